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
#include <cstring>
#include <string>
#include <vector>

#include "gem.h"
#include "gem_isa.h"

namespace {

thread_local std::string g_err;

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
  unsigned long long* bar;                  // grid barrier counter
  int* err;
  uint64_t t0;
  uint32_t ncycles, in_base, in_cap, out_cap;
  uint32_t n_stages, n_streams, state_words;
  uint32_t pi_words, po_words, q_words, cut_words, n_rams, n_flops, q_ext_words;
  uint32_t flags;
};

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

// Grid-wide barrier on a monotonically increasing 64-bit counter (reset to 0
// before each launch).  Release: bar.sync + gpu-scope fence + atomic arrive.
// Acquire: ld.acquire.gpu spin, then bar.sync.  A 10 s spin limit turns a
// deadlock (e.g. broken co-residency) into a trapped kernel instead of a hang.
__device__ __forceinline__ void grid_sync(const KParams& kp, unsigned long long& target) {
  __syncthreads();
  if (gridDim.x > 1) {
    if (threadIdx.x == 0) {
      target += gridDim.x;
      __threadfence();
      atomicAdd(kp.bar, 1ull);
      uint32_t spins = 0;
      uint64_t start = 0;
      while (ld_acquire_u64(kp.bar) < target) {
        if (++spins == 4096) start = globaltimer_ns();
        if (spins > 4096 && (spins & 4095) == 0 && globaltimer_ns() - start > 10000000000ull) {
          atomicExch(kp.err, 2);
          asm volatile("trap;");
        }
      }
    }
    __syncthreads();
  }
}

// Levels 1-5 (or 6-10) of the boomerang fold on one 32-bit word; constants are
// the packed per-unit slot words (gem_isa.h).  Bits above each level's width
// carry don't-care values that only ever shift toward higher positions.
__device__ __forceinline__ uint32_t fold5(uint32_t v, uint32_t xa, uint32_t xb, uint32_t ob) {
  uint32_t r1 = (v ^ xa) & (((v >> 16) ^ xb) | ob);
  uint32_t r2 = (r1 ^ (xa >> 16)) & (((r1 >> 8) ^ (xb >> 16)) | (ob >> 16));
  uint32_t r3 = (r2 ^ (xa >> 24)) & (((r2 >> 4) ^ (xb >> 24)) | (ob >> 24));
  uint32_t r4 = (r3 ^ (xa >> 28)) & (((r3 >> 2) ^ (xb >> 28)) | (ob >> 28));
  uint32_t r5 = (r4 ^ (xa >> 30)) & (((r4 >> 1) ^ (xb >> 30)) | (ob >> 30));
  return (r1 & 0xFFFFu) | ((r2 & 0xFFu) << 16) | ((r3 & 0xFu) << 24) | ((r4 & 3u) << 28) | ((r5 & 1u) << 30);
}

// Levels 11-13 on the 8 warp bits.
__device__ __forceinline__ uint32_t fold3(uint32_t v, uint32_t xa, uint32_t xb, uint32_t ob) {
  uint32_t r1 = (v ^ xa) & (((v >> 4) ^ xb) | ob);
  uint32_t r2 = (r1 ^ (xa >> 4)) & (((r1 >> 2) ^ (xb >> 4)) | (ob >> 4));
  uint32_t r3 = (r2 ^ (xa >> 6)) & (((r2 >> 1) ^ (xb >> 6)) | (ob >> 6));
  return (r1 & 0xFu) | ((r2 & 3u) << 4) | ((r3 & 1u) << 6);
}

__device__ __forceinline__ uint32_t rd_global(const uint32_t* p) { return __ldcg(p); }

__device__ void run_partition(const KParams& kp, uint32_t* S, uint32_t* ramp, uint32_t* topb, uint32_t p,
                              uint32_t st, uint32_t c, uint32_t cur, uint32_t nxt) {
  const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint32_t* pr = kp.prog + __ldg(kp.parts + p * GP_WORDS + GP_PROG_OFF);
  const uint4 h0 = __ldg(reinterpret_cast<const uint4*>(pr));
  const uint4 h1 = __ldg(reinterpret_cast<const uint4*>(pr) + 1);
  const uint4 h2 = __ldg(reinterpret_cast<const uint4*>(pr) + 2);
  const uint4 h3 = __ldg(reinterpret_cast<const uint4*>(pr) + 3);
  const uint32_t n_gread = h0.y, n_layers = h0.z, n_out = h0.w;
  const uint32_t n_ram = h1.x, off_gread = h1.z, off_layers = h1.w;
  const uint32_t off_out = h2.x, off_ram = h2.y, n_out_pad = h3.x;
  // ---- a2: global read of input ports (once per cycle)
  const uint32_t* gr = pr + off_gread;
  for (uint32_t k = tid; k < n_gread; k += GEM_THREADS) {
    const uint2 e = __ldg(reinterpret_cast<const uint2*>(gr) + k);
    const uint32_t reg = GEM_GID_REGION(e.x), idx = GEM_GID_INDEX(e.x);
    uint32_t v;
    if (reg == GEM_R_PI) v = __ldg(kp.pi + ((size_t)st * kp.in_cap + kp.in_base + c) * kp.pi_words + idx);
    else if (reg == GEM_R_Q) v = rd_global(kp.q + ((size_t)cur * kp.n_streams + st) * kp.q_words + idx);
    else if (reg == GEM_R_RD) v = rd_global(kp.rd + ((size_t)cur * kp.n_streams + st) * kp.n_rams + idx);
    else v = rd_global(kp.cut + (size_t)st * kp.cut_words + idx);
    S[e.y] = v;
  }
  if (tid == 0) S[0] = 0u;
  __syncthreads();
  // ---- a3-a5: layers
  const uint32_t* L = pr + off_layers;
  for (uint32_t l = 0; l < n_layers; l++) {
    const uint4 lh0 = __ldg(reinterpret_cast<const uint4*>(L));
    const uint4 n03 = __ldg(reinterpret_cast<const uint4*>(L) + 1);
    const uint4 n47 = __ldg(reinterpret_cast<const uint4*>(L) + 2);
    const uint32_t flags = lh0.y, topc = lh0.z, topwo = lh0.w;
    const uint32_t niter_all[8] = {n03.x, n03.y, n03.z, n03.w, n47.x, n47.y, n47.z, n47.w};
    const bool uses_top = (flags & GEM_LF_USES_TOP) != 0;
    if ((flags >> warp) & 1u) {
      uint32_t off = LH_WORDS;
#pragma unroll
      for (uint32_t w = 0; w < GEM_WARPS; w++)
        if (w < warp && ((flags >> w) & 1u)) off += GEM_WARP_REC_WORDS(niter_all[w]);
      const uint32_t* rec = L + off;
      uint32_t niter = 0;
#pragma unroll
      for (uint32_t w = 0; w < GEM_WARPS; w++) if (w == warp) niter = niter_all[w];
      const uint4 wc = __ldg(reinterpret_cast<const uint4*>(rec));
      const uint4 lc = __ldg(reinterpret_cast<const uint4*>(rec + 4) + lane);
      // gather (bit permutation)
      const uint32_t* lv = rec + 4 + 128 + lane;
      uint32_t v = 0;
#pragma unroll 4
      for (uint32_t i = 0; i < niter; i++) {
        const uint32_t e = __ldg(lv + i * 32);
        const uint32_t s = S[(e & 0xFFFFu) >> 5];
        v |= ((s >> (e & 31u)) & 1u) << ((e >> 16) & 31u);
      }
      // fold levels 1-5 in-thread
      const uint32_t P = fold5(v, lc.x, lc.y, lc.z);
      if (lc.w) S[lc.w] = P;
      // levels 6-10 in-warp
      const uint32_t u = __ballot_sync(0xFFFFFFFFu, (P >> 30) & 1u);
      const uint32_t Pw = fold5(u, wc.x, wc.y, wc.z);
      if (lane == 0) {
        if (wc.w) S[wc.w] = Pw;
        if (uses_top) topb[warp] = (Pw >> 30) & 1u;
      }
    } else if (uses_top && lane == 0) {
      topb[warp] = 0u;
    }
    if (uses_top) {
      __syncthreads();
      if (tid == 0) {
        uint32_t t8 = 0;
#pragma unroll
        for (uint32_t w = 0; w < GEM_WARPS; w++) t8 |= topb[w] << w;
        S[topwo] = fold3(t8, topc & 0xFFu, (topc >> 8) & 0xFFu, (topc >> 16) & 0xFFu);
      }
    }
    __syncthreads();
    L += lh0.x;
  }
  // ---- a6: endpoint commit (warp ballot-gather per output word)
  const uint32_t* od = pr + off_out;
  const uint32_t* os = od + n_out_pad;
  for (uint32_t j = warp; j < n_out; j += GEM_WARPS) {
    const uint32_t e = __ldg(os + j * 32 + lane);
    const uint32_t src = e & 0xFFFFu;
    const uint32_t bit = ((S[src >> 5] >> (src & 31u)) & 1u) ^ (e >> 31);
    const uint32_t v = __ballot_sync(0xFFFFFFFFu, bit);
    if (lane == 0) {
      const uint32_t dst = __ldg(od + j);
      const uint32_t reg = GEM_GID_REGION(dst), idx = GEM_GID_INDEX(dst);
      if (reg == GEM_R_Q) __stcg(kp.q + ((size_t)nxt * kp.n_streams + st) * kp.q_words + idx, v);
      else if (reg == GEM_R_PO) __stcg(kp.po + ((size_t)st * kp.out_cap + c) * kp.po_words + idx, v);
      else if (reg == GEM_R_CUT) __stcg(kp.cut + (size_t)st * kp.cut_words + idx, v);
      else ramp[idx] = v;
    }
  }
  // ---- a7: RAM blocks (read-first, then per-bit write; readings U7-U10)
  if (n_ram) {
    __syncthreads();
    const uint32_t* rr = pr + off_ram;
    for (uint32_t r = tid; r < n_ram; r += GEM_THREADS) {
      const uint32_t id = __ldg(rr + 4 * r);
      const uint32_t ra = ramp[4 * r + GEM_PORT_RADDR] & (GEM_RAM_WORDS - 1);
      const uint32_t wa = ramp[4 * r + GEM_PORT_WADDR] & (GEM_RAM_WORDS - 1);
      const uint32_t wd = ramp[4 * r + GEM_PORT_WDATA], be = ramp[4 * r + GEM_PORT_WBE];
      uint32_t* M = kp.mem + ((size_t)st * kp.n_rams + id) * GEM_RAM_WORDS;
      const uint32_t old = __ldcg(M + ra);
      const uint32_t cur_w = __ldcg(M + wa);
      __stcg(M + wa, (cur_w & ~be) | (wd & be));
      __stcg(kp.rd + ((size_t)nxt * kp.n_streams + st) * kp.n_rams + id, old);
    }
  }
  __syncthreads();  // S / ramp reused by the next work item
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

__global__ void __launch_bounds__(GEM_THREADS, 2) gem_step_kernel(const KParams kp) {
  extern __shared__ uint32_t smem[];
  uint32_t* S = smem;
  uint32_t* ramp = smem + kp.state_words;
  uint32_t* topb = ramp + 4 * GEM_MAX_RAMS_PER_PART;
  unsigned long long bar_target = 0;
  const bool instr = (kp.flags & (GEM_F_TRACE_STATE | GEM_F_DIGEST)) != 0;
  for (uint32_t c = 0; c < kp.ncycles; c++) {
    const uint64_t t = kp.t0 + c;
    const uint32_t cur = (uint32_t)(t & 1u), nxt = cur ^ 1u;
    if (instr && c > 0) record_state(kp, c - 1, cur);
    for (uint32_t s = 0; s < kp.n_stages; s++) {
      const uint32_t pb = __ldg(kp.stage_list + s), pe = __ldg(kp.stage_list + s + 1);
      const uint32_t np = pe - pb;
      const uint32_t n_items = np * kp.n_streams;
      for (uint32_t item = blockIdx.x; item < n_items; item += gridDim.x) {
        const uint32_t p = __ldg(kp.stage_list + kp.n_stages + 1 + pb + item % np);
        run_partition(kp, S, ramp, topb, p, item / np, c, cur, nxt);
      }
      grid_sync(kp, bar_target);
    }
  }
  if (instr) record_state(kp, kp.ncycles - 1, (uint32_t)((kp.t0 + kp.ncycles) & 1u));
}

// external <-> internal layout conversion kernels
// out[st][row][ext_w] = gather of 32 internal bits via int_of_ext
__global__ void unpermute_kernel(const uint32_t* __restrict__ in, uint32_t* __restrict__ out,
                                 const uint32_t* __restrict__ int_of_ext, uint32_t n_bits, uint32_t in_words,
                                 uint32_t out_words, uint64_t rows, uint64_t in_row_stride,
                                 uint64_t out_row_stride) {
  const uint64_t total = rows * out_words;
  for (uint64_t g = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; g < total;
       g += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t row = g / out_words;
    const uint32_t w = (uint32_t)(g % out_words);
    const uint32_t* src = in + row * in_row_stride;
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
  // device buffers
  uint32_t *d_prog = nullptr, *d_parts = nullptr, *d_stage = nullptr;
  uint32_t *d_q_int_of_ext = nullptr, *d_q_ext_of_int = nullptr, *d_po_int_of_ext = nullptr;
  uint32_t *d_q = nullptr, *d_rd = nullptr, *d_cut = nullptr, *d_mem = nullptr;
  uint32_t *d_pi = nullptr, *d_po = nullptr, *d_qtrace = nullptr, *d_scratch = nullptr;
  unsigned long long *d_digest = nullptr, *d_bar = nullptr;
  int* d_err = nullptr;
  uint32_t in_cap = 0, in_queued = 0, in_head = 0, out_cap = 0, last_cycles = 0;
  size_t scratch_bytes = 0;
  uint64_t cycle = 0;
  cudaEvent_t ev0 = nullptr, ev1 = nullptr;
  float last_ms = 0.f;
};

static int fail(int code, const std::string& msg) {
  g_err = msg;
  return code;
}

#define CK(call)                                                                          \
  do {                                                                                    \
    cudaError_t e_ = (call);                                                              \
    if (e_ != cudaSuccess) {                                                              \
      if (sim) sim->poisoned = true;                                                      \
      return fail(e_ == cudaErrorMemoryAllocation ? GEM_E_NOMEM : GEM_E_CUDA,             \
                  std::string(#call) + ": " + cudaGetErrorString(e_));                    \
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
  uint32_t cap = std::max<uint32_t>(ncycles, 16);
  if (sim->d_po) cudaFree(sim->d_po);
  if (sim->d_qtrace) cudaFree(sim->d_qtrace);
  if (sim->d_digest) cudaFree(sim->d_digest);
  sim->d_po = nullptr; sim->d_qtrace = nullptr; sim->d_digest = nullptr;
  sim->out_cap = 0;
  CK(dalloc(&sim->d_po, (size_t)sim->n_streams * cap * sim->po_words_int * 4));
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

extern "C" {

const char* gem_last_error(void) { return g_err.c_str(); }

int gem_load_program(const void* blob, size_t nbytes, const gem_config* cfg, gem_sim** out) {
  gem_sim* sim = nullptr;
  if (!blob || !cfg || !out || nbytes < GH_N_WORDS * 4 || (nbytes & 3)) return fail(GEM_E_INVAL, "bad arguments");
  const uint32_t* w = (const uint32_t*)blob;
  const size_t nw = nbytes / 4;
  if (w[GH_MAGIC] != GEM_MAGIC || w[GH_VERSION] != GEM_VERSION) return fail(GEM_E_FORMAT, "bad blob magic/version");
  const uint64_t total_words = w[GH_TOTAL_WORDS_LO] | ((uint64_t)w[GH_TOTAL_WORDS_HI] << 32);
  const uint64_t prog_words = w[GH_PROG_WORDS_LO] | ((uint64_t)w[GH_PROG_WORDS_HI] << 32);
  if (total_words != nw || w[GH_OFF_PROG] + prog_words > nw) return fail(GEM_E_FORMAT, "truncated blob");
  if (cfg->n_streams == 0) return fail(GEM_E_INVAL, "n_streams must be >= 1");
  if (w[GH_MAX_STATE_WORDS] > GEM_MAX_STATE_WORDS) return fail(GEM_E_FORMAT, "state too large");
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0)
    return fail(GEM_E_UNSUPPORTED, "no CUDA device (libgem has no CPU fallback)");
  if (cfg->device < 0 || cfg->device >= ndev) return fail(GEM_E_INVAL, "bad device ordinal");
  sim = new gem_sim();
  *out = nullptr;
  sim->device = cfg->device;
  sim->flags = cfg->flags;
  sim->n_streams = cfg->n_streams;
  {
    cudaError_t e = cudaSetDevice(sim->device);
    if (e != cudaSuccess) { delete sim; return fail(GEM_E_CUDA, cudaGetErrorString(e)); }
  }
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
    if (pr[PH_MAGIC] != GEM_PART_MAGIC || pr[PH_N_RAM] > GEM_MAX_RAMS_PER_PART) {
      delete sim;
      return fail(GEM_E_FORMAT, "bad partition program");
    }
  }
  // inverse permutation tables
  std::vector<uint32_t> q_int_of_ext(std::max<uint32_t>(sim->n_flops, 1), 0),
      po_int_of_ext(std::max<uint32_t>(sim->n_po, 1), 0);
  for (uint32_t b = 0; b < sim->q_words_int * 32; b++)
    if (q_ext_of_int[b] != 0xFFFFFFFFu) q_int_of_ext[q_ext_of_int[b]] = b;
  for (uint32_t b = 0; b < sim->po_words_int * 32; b++)
    if (po_ext_of_int[b] != 0xFFFFFFFFu) po_int_of_ext[po_ext_of_int[b]] = b;
  // streams / events
  if (cfg->cuda_stream) sim->stream = (cudaStream_t)cfg->cuda_stream;
  else { CK(cudaStreamCreateWithFlags(&sim->stream, cudaStreamNonBlocking)); sim->own_stream = true; }
  CK(cudaEventCreate(&sim->ev0));
  CK(cudaEventCreate(&sim->ev1));
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
  CK(dalloc(&sim->d_q, 2 * S * sim->q_words_int * 4));
  CK(dalloc(&sim->d_rd, 2 * S * std::max<uint32_t>(sim->n_rams, 1) * 4));
  CK(dalloc(&sim->d_cut, S * std::max<uint32_t>(sim->cut_words, 1) * 4));
  CK(dalloc(&sim->d_mem, S * sim->n_rams * (size_t)GEM_RAM_WORDS * 4));
  CK(dalloc(&sim->d_bar, 64));
  CK(dalloc(&sim->d_err, 64));
  CK(cudaMemset(sim->d_err, 0, 64));
  // initial state: flops = init (U5), RD = 0, RAM = 0 (U10)
  {
    std::vector<uint32_t> q0(S * sim->q_words_int);
    for (size_t s = 0; s < S; s++) std::memcpy(&q0[s * sim->q_words_int], finit, sim->q_words_int * 4);
    CK(cudaMemcpy(sim->d_q, q0.data(), q0.size() * 4, cudaMemcpyHostToDevice));
    CK(cudaMemset(sim->d_q + S * sim->q_words_int, 0, S * sim->q_words_int * 4));
    CK(cudaMemset(sim->d_rd, 0, 2 * S * std::max<uint32_t>(sim->n_rams, 1) * 4));
    CK(cudaMemset(sim->d_cut, 0, S * std::max<uint32_t>(sim->cut_words, 1) * 4));
    if (sim->n_rams) CK(cudaMemset(sim->d_mem, 0, S * sim->n_rams * (size_t)GEM_RAM_WORDS * 4));
  }
  // persistent co-resident grid
  sim->smem_bytes = (sim->state_words + 4 * GEM_MAX_RAMS_PER_PART + GEM_WARPS) * 4;
  if (sim->smem_bytes > 48 * 1024)
    CK(cudaFuncSetAttribute(gem_step_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sim->smem_bytes));
  int bps = 0, sms = 0, coop = 0;
  CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&bps, gem_step_kernel, GEM_THREADS, sim->smem_bytes));
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, sim->device));
  CK(cudaDeviceGetAttribute(&coop, cudaDevAttrCooperativeLaunch, sim->device));
  if (bps < 1 || !coop) { gem_free(sim); return fail(GEM_E_UNSUPPORTED, "kernel cannot be made co-resident"); }
  sim->blocks_per_sm = (uint32_t)bps;
  sim->sm_count = (uint32_t)sms;
  uint32_t cap = (uint32_t)bps * (uint32_t)sms;
  sim->grid = std::max<uint32_t>(1, std::min(cap, sim->max_items));
  if (cfg->grid_limit) sim->grid = std::max<uint32_t>(1, std::min(sim->grid, cfg->grid_limit));
  CK(cudaDeviceSynchronize());
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
    sim->in_cap = cap;
  }
  if (ncycles && sim->pi_words) {
    const size_t row = (size_t)ncycles * sim->pi_words * 4;
    CK(cudaMemcpy2DAsync(sim->d_pi, (size_t)sim->in_cap * sim->pi_words * 4, pi, row, row, sim->n_streams,
                         src_on_device ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice, sim->stream));
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
  CK(cudaMemsetAsync(sim->d_bar, 0, 8, sim->stream));
  if (sim->flags & GEM_F_DIGEST)
    CK(cudaMemsetAsync(sim->d_digest, 0, (size_t)sim->n_streams * sim->out_cap * 8, sim->stream));
  void* args[] = {&kp};
  CK(cudaEventRecord(sim->ev0, sim->stream));
  CK(cudaLaunchCooperativeKernel((const void*)gem_step_kernel, dim3(sim->grid), dim3(GEM_THREADS), args,
                                 sim->smem_bytes, sim->stream));
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
  // rows = stream*ncycles + cycle; in-row stride = po_words_int, with stream stride out_cap
  for (uint32_t s = 0; s < sim->n_streams; s++) {
    unpermute_kernel<<<std::min<uint64_t>(4096, (ncycles * sim->po_words_ext + 255) / 256 + 1), 256, 0,
                       sim->stream>>>(sim->d_po + (size_t)s * sim->out_cap * sim->po_words_int,
                                      out + (size_t)s * ncycles * sim->po_words_ext, sim->d_po_int_of_ext,
                                      sim->n_po, sim->po_words_int, sim->po_words_ext, ncycles,
                                      sim->po_words_int, sim->po_words_ext);
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
  uint32_t* out = dst;
  if (!dst_on_device) {
    if (int r = ensure_scratch(sim, bytes)) return r;
    out = sim->d_scratch;
  }
  unpermute_kernel<<<std::min<uint64_t>(4096, ((uint64_t)sim->n_streams * sim->q_words_ext + 255) / 256 + 1), 256,
                     0, sim->stream>>>(sim->d_q + (size_t)buf * sim->n_streams * sim->q_words_int, out,
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
  permute_kernel<<<std::min<uint64_t>(4096, ((uint64_t)sim->n_streams * sim->q_words_int + 255) / 256 + 1), 256, 0,
                   sim->stream>>>(sim->d_scratch, sim->d_q + (size_t)buf * sim->n_streams * sim->q_words_int,
                                  sim->d_q_ext_of_int, sim->q_words_int, sim->q_words_ext, sim->n_streams);
  CK(cudaGetLastError());
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

void gem_free(gem_sim* sim) {
  if (!sim) return;
  cudaSetDevice(sim->device);
  if (sim->stream) cudaStreamSynchronize(sim->stream);
  for (void* p : {(void*)sim->d_prog, (void*)sim->d_parts, (void*)sim->d_stage, (void*)sim->d_q_int_of_ext,
                  (void*)sim->d_q_ext_of_int, (void*)sim->d_po_int_of_ext, (void*)sim->d_q, (void*)sim->d_rd,
                  (void*)sim->d_cut, (void*)sim->d_mem, (void*)sim->d_pi, (void*)sim->d_po, (void*)sim->d_qtrace,
                  (void*)sim->d_scratch, (void*)sim->d_digest, (void*)sim->d_bar, (void*)sim->d_err})
    if (p) cudaFree(p);
  if (sim->ev0) cudaEventDestroy(sim->ev0);
  if (sim->ev1) cudaEventDestroy(sim->ev1);
  if (sim->own_stream && sim->stream) cudaStreamDestroy(sim->stream);
  delete sim;
}

}  // extern "C"
