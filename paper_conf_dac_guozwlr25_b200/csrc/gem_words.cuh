// gem_words.cuh -- word mode: the single-stream latency path (gem_isa.h "WRD1").
// Included by gem_runtime.cu after gem_lanes.cuh (uses KParams, grid_sync,
// record_state, the TMA / mbarrier helpers and the work-list layout).
//
// Per simulated cycle, for each stage s, each CTA runs its work items
// (partition p, stream st) of stage s:
//   a1/a2  input ports: entry k = one global bit (PI[t] / Q_cur / RD_cur /
//          stage cut), stored as word 1 + k of the partition state S (P:196
//          "only once per cycle")
//   a3-a5  the partition's ANDs in barrier-separated steps: thread t runs ops
//          t, t + 256, ... of the step, each two LDS, two LOP3, one STS; a
//          step's operands were written in earlier steps (P:81 AND/inverter
//          graph, evaluated in the paper's dependency order)
//   a6     endpoint commit: warp ballot of 32 endpoint bits per owned output
//          word -> Q_next / PO[t] / CUT / RAM-port staging
//   a7     RAM blocks: read-first, then per-bit write (readings U7-U10)
//   a8     grid barrier per stage
// Every program a CTA runs is copied into its shared memory once per launch
// (TMA bulk copy); the host plans word mode only when that fits.
// Why words instead of the bit-packed boomerang layer for one stream:
// DESIGN.md sec. 8d (measured: a layer ~1.6K clk advances the critical path by
// ~6 levels; a step ~0.12K clk advances it by one).

#define GEM_WORD_RAMP (4 * GEM_MAX_RAMS_PER_PART)
#ifndef GEM_WORD_THREADS
#define GEM_WORD_THREADS 256   /* threads of a word-mode CTA (a step's round) */
#endif
#define GEM_WORD_WARPS (GEM_WORD_THREADS / 32)
#define GEM_WORD_PORT_REGS 4   /* port entries per thread kept in registers (fast path) */

// Header fields of a word program (loaded once per launch on the fast path).
struct WordHdr {
  uint32_t n_gread, n_steps, n_out, n_ram, off_steps, off_ops, off_out, off_ram, off_gread;
};
__device__ __forceinline__ WordHdr word_hdr(const uint32_t* P) {
  const uint4 h0 = *reinterpret_cast<const uint4*>(P);
  const uint4 h1 = *(reinterpret_cast<const uint4*>(P) + 1);
  const uint4 h2 = *(reinterpret_cast<const uint4*>(P) + 2);
  return WordHdr{h0.y, h0.z, h1.x, h1.y, h1.w, h2.x, h2.y, h2.z, h2.w};
}
// Fast path (a CTA with one work item per cycle and <= 1024 ports): each
// thread keeps its port gids in registers and loads its PI words of cycle c+1
// during cycle c (their HBM latency hides behind the steps).
struct WordPorts {
  uint32_t g[GEM_WORD_PORT_REGS];
  uint32_t pv[GEM_WORD_PORT_REGS];
};

__device__ __forceinline__ uint2 lds64(uint32_t addr) {
  uint2 r;
  asm volatile("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(r.x), "=r"(r.y) : "r"(addr));
  return r;
}
// one AND: S[y] = (S[a] ^ ia) & (S[b] ^ ib) on bit 0 (gem_isa.h WRD1 op)
__device__ __forceinline__ void word_op(uint32_t s_base, uint2 o) {
  const uint32_t a = lds(s_base + (o.x & 0xFFFCu)), b = lds(s_base + ((o.x >> 16) & 0xFFFCu));
  sts(s_base + o.y, (a ^ o.x) & (b ^ (o.x >> 16)));
}
// The same with S at shared-window address GEM_S0_ADDR (the start of dynamic
// shared memory, checked by the caller): the byte offsets address S through
// the load/store immediate, no add on the step's dependency chain; o = {0, 0}
// (no op) reads word 0 and stores nothing (predicated, no branch).
__device__ __forceinline__ uint32_t lds_s0(uint32_t off) {
  uint32_t v;
  asm volatile("ld.shared.u32 %0, [%1+1024];" : "=r"(v) : "r"(off));
  return v;
}
__device__ __forceinline__ void word_op_s0(uint2 o) {
  const uint32_t a = lds_s0(o.x & 0xFFFCu), b = lds_s0((o.x >> 16) & 0xFFFCu);
  const uint32_t r = (a ^ o.x) & (b ^ (o.x >> 16));
  asm volatile("{\n .reg .pred p;\n setp.ne.u32 p, %0, 0;\n @p st.shared.u32 [%0+1024], %1;\n}" ::"r"(o.y), "r"(r)
               : "memory");
}
// Global word of input port gid g (region << 24 | bit) for stream st, cycle c.
template <bool LOC>
__device__ __forceinline__ uint32_t port_word(const KParams& kp, uint32_t g, uint32_t st, uint32_t c, uint32_t cur,
                                              const uint32_t* loc) {
  const uint32_t reg = g >> 24, wi = (g & 0xFFFFFFu) >> 5;
  if (reg == GEM_R_Q)
    return LOC ? loc[cur * kp.loc_words + wi] : rd_global(kp.q + ((size_t)cur * kp.n_streams + st) * kp.q_words + wi);
  if (reg == GEM_R_PI) return rd_global(kp.pi + ((size_t)st * kp.in_cap + kp.in_base + c) * kp.pi_words + wi);
  if (reg == GEM_R_RD)
    return LOC ? loc[cur * kp.loc_words + kp.q_words + wi]
               : rd_global(kp.rd + ((size_t)cur * kp.n_streams + st) * kp.n_rams + wi);
  return rd_global(kp.cut + (size_t)st * kp.cut_words + wi);
}

// One work item (partition program P, stream st, cycle c).  FAST: ports in
// registers + PI prefetch (wp), see WordPorts.
template <bool LOC, bool FAST>
__device__ __forceinline__ void run_word_partition(const KParams& kp, const uint32_t* P, const WordHdr& H,
                                                   WordPorts& wp, uint32_t s_base, uint32_t* ramp, uint32_t st,
                                                   uint32_t c, uint32_t cur, uint32_t nxt, bool prof_on,
                                                   uint32_t* loc) {
  const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  PROF(7);
  // ---- a1/a2: input ports (bit 0 of word 1 + k = port k)
  if (FAST) {
    uint32_t v[GEM_WORD_PORT_REGS];
#pragma unroll
    for (uint32_t u = 0; u < GEM_WORD_PORT_REGS; u++) {
      const uint32_t g = wp.g[u];
      v[u] = 0u;
      if (g != ~0u) v[u] = ((g >> 24) == GEM_R_PI && c > 0) ? wp.pv[u] : port_word<LOC>(kp, g, st, c, cur, loc);
    }
#pragma unroll
    for (uint32_t u = 0; u < GEM_WORD_PORT_REGS; u++)
      if (wp.g[u] != ~0u) sts(s_base + 4u * (1u + u * GEM_WORD_THREADS + tid), v[u] >> (wp.g[u] & 31u));
    // next cycle's PI words (consumed at the top of cycle c+1)
#pragma unroll
    for (uint32_t u = 0; u < GEM_WORD_PORT_REGS; u++)
      if (wp.g[u] != ~0u && (wp.g[u] >> 24) == GEM_R_PI && c + 1 < kp.ncycles)
        wp.pv[u] = port_word<LOC>(kp, wp.g[u], st, c + 1, cur, loc);
  } else {
    const uint32_t* gr = P + H.off_gread;
    constexpr uint32_t GU = 4;
    for (uint32_t k0 = 0; k0 < H.n_gread; k0 += GU * GEM_WORD_THREADS) {
      uint32_t v[GU], sh[GU];
#pragma unroll
      for (uint32_t u = 0; u < GU; u++) {
        const uint32_t k = k0 + u * GEM_WORD_THREADS + tid;
        v[u] = 0u;
        sh[u] = 0u;
        if (k < H.n_gread) {
          const uint32_t g = gr[k];
          sh[u] = g & 31u;
          v[u] = port_word<LOC>(kp, g, st, c, cur, loc);
        }
      }
#pragma unroll
      for (uint32_t u = 0; u < GU; u++) {
        const uint32_t k = k0 + u * GEM_WORD_THREADS + tid;
        if (k < H.n_gread) sts(s_base + 4u * (1u + k), v[u] >> sh[u]);
      }
    }
  }
  PROF(8);
  if (tid == 0) sts(s_base, 0u);
  __syncthreads();
  PROF(1);
  // ---- a3-a5: steps.  A step has n <= 4 x 256 ops (the host checks); thread t
  // runs ops t, t + 256, ... < n.  Latency layout (scripts/ubench_steps2.cu:
  // ~110-130 clk per step against ~300 for a loop that prepares addresses or
  // loads bounds ahead of its operand loads): after the barrier a thread issues
  // its operand loads first, then the loads of later steps' bounds and op
  // words; the first-round op of a step is in a register before the step
  // begins, rounds 1-3 (the capacity-bound wide steps) are loaded in the step.
  const uint32_t* stp = P + H.off_steps;
  const uint32_t o_base = smem_u32(P + H.off_ops) + 8u * tid;
  const uint32_t ns = H.n_steps;
  auto bound = [&](uint32_t k) { return stp[min(k, ns)]; };
  if (s_base == GEM_S0_ADDR) {
    // op words two steps ahead (o: this step, o1: the next one, loaded during
    // the previous step), bounds e0..e3 of steps s..s+3 in registers, e4
    // loaded during the step: whatever the compiler hoists above a barrier
    // only touches values that arrived a step earlier (one step ahead, every
    // other step of an unrolled pair waited ~80 clk at the barrier for its
    // op load)
    uint32_t e0 = 0, e1 = 0, e2 = 0, e3 = 0;
    uint2 o = make_uint2(0u, 0u), o1 = o;
    if (ns) {
      e1 = bound(1);
      e2 = bound(2);
      e3 = bound(3);
      if (tid < e1) o = lds64(o_base);
      if (tid < e2 - e1) o1 = lds64(o_base + 8u * e1);
    }
    // unrolled by 4 (measured: C3 122.9K cycles/s vs 120.7K at the compiler's
    // 2, 118.5K at 1, 116.7K at 8; the copies of an unrolled loop schedule
    // differently and a barrier-bound loop pays for the slowest)
#pragma unroll 4
    for (uint32_t s = 0; s < ns; s++) {
      // loads whose results are consumed a step later go first (their latency
      // then never meets a barrier: a value loaded just before the barrier and
      // used right after it stalls the in-order issue of the next step)
      const uint32_t e4 = bound(s + 4);
      uint2 o2 = make_uint2(0u, 0u);
      if (tid < e3 - e2) o2 = lds64(o_base + 8u * e2);
      word_op_s0(o);
      const uint32_t n = e1 - e0;
      if (n > GEM_WORD_THREADS) {   // CTA-uniform: rounds 1-3 of a wide step
        uint2 w[3];
#pragma unroll
        for (uint32_t r = 0; r < 3; r++) {
          w[r] = make_uint2(0u, 0u);
          if (tid + (r + 1) * GEM_WORD_THREADS < n) w[r] = lds64(o_base + 8u * (e0 + (r + 1) * GEM_WORD_THREADS));
        }
#pragma unroll
        for (uint32_t r = 0; r < 3; r++) word_op_s0(w[r]);
      }
      o = o1;
      o1 = o2;
      e0 = e1;
      e1 = e2;
      e2 = e3;
      e3 = e4;
      __syncthreads();
    }
  } else {
    uint32_t e0 = 0, e1 = 0, e2 = 0;
    uint2 o = make_uint2(0u, 0u);
    bool v = false;
    if (ns) {
      e1 = bound(1);
      e2 = bound(2);
      v = tid < e1;
      if (v) o = lds64(o_base);
    }
    for (uint32_t s = 0; s < ns; s++) {
      if (v) word_op(s_base, o);
      const uint32_t n = e1 - e0;
      for (uint32_t r = 1; r < 4; r++)
        if (tid + r * GEM_WORD_THREADS < n) word_op(s_base, lds64(o_base + 8u * (e0 + r * GEM_WORD_THREADS)));
      const uint32_t e3 = bound(s + 3);
      v = tid < e2 - e1;
      if (v) o = lds64(o_base + 8u * e1);
      e0 = e1;
      e1 = e2;
      e2 = e3;
      __syncthreads();
    }
  }
  PROF(2);
  // ---- a6: endpoint commit (one warp ballot per owned output word)
  const uint32_t* od = P + H.off_out;
  const uint32_t* os = od + H.n_out;
  for (uint32_t o = warp; o < H.n_out; o += GEM_WORD_WARPS) {
    const uint32_t e = os[o * 32 + lane];
    const uint32_t bit = (lds(s_base + (e & 0xFFFCu)) ^ e) & 1u;
    const uint32_t v = __ballot_sync(0xFFFFFFFFu, bit);
    if (lane == 0) {
      const uint32_t dst = od[o];
      const uint32_t reg = GEM_GID_REGION(dst), idx = GEM_GID_INDEX(dst);
      if (reg == GEM_R_Q) {
        __stcg(kp.q + ((size_t)nxt * kp.n_streams + st) * kp.q_words + idx, v);
        if (LOC) loc[nxt * kp.loc_words + idx] = v;
      } else if (reg == GEM_R_PO) {
        __stcg(kp.po + ((size_t)st * kp.out_cap + c) * kp.po_words + idx, v);
      } else if (reg == GEM_R_CUT) {
        __stcg(kp.cut + (size_t)st * kp.cut_words + idx, v);
      } else {
        ramp[idx] = v;
      }
    }
  }
  // ---- a7: RAM blocks (read-first, then per-bit write)
  if (H.n_ram) {
    __syncthreads();
    const uint32_t* rr = P + H.off_ram;
    for (uint32_t r = tid; r < H.n_ram; r += GEM_WORD_THREADS) {
      const uint32_t* rp = ramp + 4 * r;
      const uint32_t id = rr[4 * r];
      const uint32_t ra = rp[GEM_PORT_RADDR] & (GEM_RAM_WORDS - 1);
      const uint32_t wa = rp[GEM_PORT_WADDR] & (GEM_RAM_WORDS - 1);
      const uint32_t wd = rp[GEM_PORT_WDATA], be = rp[GEM_PORT_WBE];
      uint32_t* M = kp.mem + ((size_t)st * kp.n_rams + id) * GEM_RAM_WORDS;
      const uint32_t old = __ldcg(M + ra);
      const uint32_t cur_w = __ldcg(M + wa);
      __stcg(M + wa, (cur_w & ~be) | (wd & be));
      __stcg(kp.rd + ((size_t)nxt * kp.n_streams + st) * kp.n_rams + id, old);
      if (LOC) loc[nxt * kp.loc_words + kp.q_words + id] = old;
    }
  }
  __syncthreads();   // S / ramp reused by the next work item
  PROF(3);
}

// LOC: single-CTA launch of one stream (every flop and RAM-read word is
// written by this CTA), so Q / RD are read from a shared-memory copy.
template <bool LOC>
__global__ void __launch_bounds__(GEM_WORD_THREADS, 1) gem_word_kernel(const KParams kp) {
  extern __shared__ __align__(16) uint32_t smem[];
  // layout (words): S[state_words] | area[area_words] | ramp[GEM_WORD_RAMP] | res_p[16] | res_off[16] |
  //                 res_n[16] | wl cache | mbar[2 x u64] | loc[2][loc_words]
  uint32_t* S = smem;
  uint32_t* area = S + kp.state_words;
  uint32_t* ramp = area + kp.area_words;
  uint32_t* res_p = ramp + GEM_WORD_RAMP;
  uint32_t* res_off = res_p + GEM_MAX_RESIDENT;
  uint32_t* res_n = res_off + GEM_MAX_RESIDENT;
  uint32_t* wlc = res_n + 16;
  uint64_t* mbar = reinterpret_cast<uint64_t*>(wlc + GEM_WL_CACHE_WORDS);
  uint32_t* loc = reinterpret_cast<uint32_t*>(mbar + 2);
  const uint32_t tid = threadIdx.x;
  const uint32_t G = gridDim.x, B = blockIdx.x;
  const uint32_t s_base = smem_u32(S);
  if (tid == 0) {
    // the CTA's work list (fixed for the launch) into shared memory, and every
    // distinct program of it into the area (the host checked that it fits)
    uint32_t n = 0, np = 0, words = 0;
    for (uint32_t s = 0; s < kp.n_stages; s++) {
      const uint32_t b = __ldg(kp.wl_off + s * (G + 1) + B), e = __ldg(kp.wl_off + s * (G + 1) + B + 1);
      wlc[s] = b;
      wlc[8 + s] = e;
      wlc[16 + s] = n;
      for (uint32_t k = b; k < e; k++) {
        const uint2 it = __ldg(&kp.wl_items[k]);
        reinterpret_cast<uint2*>(wlc + 32)[n++] = it;
        bool seen = false;
        for (uint32_t j = 0; j < np; j++) seen |= res_p[j] == it.x;
        if (!seen) {
          res_p[np] = it.x;
          res_off[np] = words;
          words += __ldg(kp.lprog + __ldg(kp.parts + it.x * GP_WORDS + GP_WORD_OFF) + WPH_PROG_LEN);
          np++;
        }
      }
    }
    res_n[0] = np;
    res_n[1] = n;
    mbar_init(mbar, 1);
    fence_mbar_init();
    if (words) {
      mbar_expect_tx(mbar, words * 4);
      for (uint32_t j = 0; j < np; j++) {
        const uint32_t* g = kp.lprog + __ldg(kp.parts + res_p[j] * GP_WORDS + GP_WORD_OFF);
        tma_load_1d(area + res_off[j], g, __ldg(g + WPH_PROG_LEN) * 4, mbar);
      }
    }
  }
  __syncthreads();
  const uint32_t n_res = res_n[0], n_items = res_n[1];
  if (n_res) mbar_wait(mbar, 0);
  if (LOC) {
    const uint32_t c0 = (uint32_t)(kp.t0 & 1u);
    for (uint32_t k = tid; k < kp.loc_words; k += GEM_WORD_THREADS)
      loc[c0 * kp.loc_words + k] = k < kp.q_words ? __ldcg(kp.q + (size_t)c0 * kp.n_streams * kp.q_words + k)
                                                  : __ldcg(kp.rd + (size_t)c0 * kp.n_streams * kp.n_rams + (k - kp.q_words));
    __syncthreads();
  }
  unsigned long long bar_target = 0;
  const bool instr = (kp.flags & (GEM_F_TRACE_STATE | GEM_F_DIGEST)) != 0;
  WordPorts wp;
  // fast path: one stage, one work item, <= 1024 ports (every per-cycle constant
  // in registers; C1-C3 single stream)
  const WordHdr H1 = word_hdr(area);
  const bool fast = kp.n_stages == 1 && n_items == 1 && H1.n_gread <= GEM_WORD_PORT_REGS * GEM_WORD_THREADS;
  if (fast) {
    const uint2 it = reinterpret_cast<const uint2*>(wlc + 32)[0];
#pragma unroll
    for (uint32_t u = 0; u < GEM_WORD_PORT_REGS; u++) {
      const uint32_t k = u * GEM_WORD_THREADS + tid;
      wp.g[u] = k < H1.n_gread ? area[H1.off_gread + k] : ~0u;
      wp.pv[u] = 0u;
    }
    for (uint32_t c = 0; c < kp.ncycles; c++) {
      const uint64_t t = kp.t0 + c;
      const uint32_t cur = (uint32_t)(t & 1u), nxt = cur ^ 1u;
      if (instr && c > 0) record_state(kp, c - 1, cur);
      const bool prof_on = kp.prof && c < kp.prof_cycles;
      PROF(0);
      run_word_partition<LOC, true>(kp, area, H1, wp, s_base, ramp, it.y, c, cur, nxt, prof_on, loc);
      if (prof_on && tid == 0) {
        kp.prof[((size_t)c * gridDim.x + blockIdx.x) * GEM_PROF_SLOTS + 6] = H1.n_steps;
        kp.prof[((size_t)c * gridDim.x + blockIdx.x) * GEM_PROF_SLOTS + 10] = it.x;
      }
      PROF(4);
      grid_sync(kp, bar_target);
      PROF(5);
    }
  } else {
    for (uint32_t c = 0; c < kp.ncycles; c++) {
      const uint64_t t = kp.t0 + c;
      const uint32_t cur = (uint32_t)(t & 1u), nxt = cur ^ 1u;
      if (instr && c > 0) record_state(kp, c - 1, cur);
      const bool prof_on = kp.prof && c < kp.prof_cycles;
      PROF(0);
      for (uint32_t s = 0; s < kp.n_stages; s++) {
        const uint32_t kb = wlc[s], ke = wlc[8 + s];
        for (uint32_t k = kb; k < ke; k++) {
          const uint2 it = reinterpret_cast<const uint2*>(wlc + 32)[wlc[16 + s] + (k - kb)];
          uint32_t off = 0;
          for (uint32_t j = 0; j < n_res; j++) if (res_p[j] == it.x) off = res_off[j];
          const bool pr = prof_on && k == kb && s == 0;
          const WordHdr H = word_hdr(area + off);
          run_word_partition<LOC, false>(kp, area + off, H, wp, s_base, ramp, it.y, c, cur, nxt, pr, loc);
          if (pr && tid == 0) {
            kp.prof[((size_t)c * gridDim.x + blockIdx.x) * GEM_PROF_SLOTS + 6] = H.n_steps;
            kp.prof[((size_t)c * gridDim.x + blockIdx.x) * GEM_PROF_SLOTS + 10] = it.x;
          }
        }
        if (s == 0) PROF(4);
        grid_sync(kp, bar_target);
      }
      PROF(5);
    }
  }
  if (instr) record_state(kp, kp.ncycles - 1, (uint32_t)((kp.t0 + kp.ncycles) & 1u));
}
