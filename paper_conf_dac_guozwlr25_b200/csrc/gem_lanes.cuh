// gem_lanes.cuh -- lane mode: stream-sliced execution of the same VLIW
// placement for batched stimulus streams.
// Included by gem_runtime.cu (shares KParams and the grid barrier).
//
// Every signal of a 32-stream group is one 32-bit lane word (bit s = stream s),
// so one pass over a boomerang layer evaluates it for 32
// streams: a leaf is one shared-memory load of a whole word (no bit
// extraction) and each gate slot is (A ^ XA) & ((B ^ XB) | OB) on words, with
// XA/XB/OB the slot's constants sign-extended to masks.  The program
// (gem_isa.h "Lane mode") comes from the same placement as the bit-packed one.

// lane global-state indexing, group-minor: X[row][bit][group] (row = buffer
// parity or cycle).  The K groups of a work item are adjacent words, so a port
// load or an endpoint store of all K groups is one 16-byte access for K = 4.
struct LaneIdx {
  uint32_t G;
  __device__ __forceinline__ size_t q(uint32_t buf, uint32_t bits, uint32_t b, uint32_t g) const {
    return ((size_t)buf * bits + b) * G + g;
  }
};

// one lane layer's per-thread records (loaded before the previous layer's barrier)
struct LaneRegs {
  uint4 e[4];                 // 32 u16 leaf lane words
  uint4 lc;                   // xa, xb, ob, write mask (levels 1-5)
  uint32_t base;              // write-out base lane word
  uint4 wc;                   // wxa, wxb, wob, wmask (levels 6-10)
  uint32_t wbase;
  uint32_t flags, topc, topwo, size;           // this layer's header
  uint32_t nflags, ntopc, ntopwo, nsize, nwoff;  // the next layer's (LLH_NEXT copy)
};

// Records come straight from global memory (L2-resident program; no shared
// memory ring): every warp loads its own record, one layer ahead of its use.
__device__ __forceinline__ void load_lane_rec(const uint32_t* rec, LaneRegs& R) {
  const uint32_t lane = threadIdx.x & 31;
  R.wc = __ldg(reinterpret_cast<const uint4*>(rec));
  R.wbase = __ldg(rec + 4);
  R.lc = __ldg(reinterpret_cast<const uint4*>(rec + GEM_LWREC_HDR) + lane);
  const uint4* lv = reinterpret_cast<const uint4*>(rec + GEM_LWREC_LEAVES) + lane;
#pragma unroll
  for (uint32_t g = 0; g < 4; g++) R.e[g] = __ldg(lv + g * 32);
  R.base = __ldg(rec + GEM_LWREC_BASE + lane);
}
__device__ __forceinline__ void take_next_header(const uint32_t* L, LaneRegs& R) {
  const uint4 n = __ldg(reinterpret_cast<const uint4*>(L + LLH_NEXT));
  R.nwoff = __ldg(L + LLH_NEXT + LLH_WOFF0 + (threadIdx.x >> 5));
  R.nsize = n.x;
  R.nflags = n.y;
  R.ntopc = n.z;
  R.ntopwo = n.w;
}
// layer 0 of an item: its header, then its records (one dependent step)
__device__ __forceinline__ void load_lane_first(const uint32_t* L, LaneRegs& R) {
  const uint32_t warp = threadIdx.x >> 5;
  const uint4 h = __ldg(reinterpret_cast<const uint4*>(L));
  const uint32_t woff = __ldg(L + LLH_WOFF0 + warp);
  take_next_header(L, R);
  R.size = h.x;
  R.flags = h.y;
  R.topc = h.z;
  R.topwo = h.w;
  if ((R.flags >> warp) & 1u) load_lane_rec(L + woff, R);
}
// layer l+1 at L: its header is already in R.n*, so its records and the header
// of layer l+2 are all loaded at once
__device__ __forceinline__ void load_lane_next(const uint32_t* L, LaneRegs& R) {
  const uint32_t warp = threadIdx.x >> 5;
  R.size = R.nsize;
  R.flags = R.nflags;
  R.topc = R.ntopc;
  R.topwo = R.ntopwo;
  const uint32_t woff = R.nwoff;
  take_next_header(L, R);
  if ((R.flags >> warp) & 1u) load_lane_rec(L + woff, R);
}

// K-word vectors: a work item runs K 32-stream groups together, their lane
// words interleaved in shared memory (word w of group j at S[w*K + j]) so a
// leaf is one LDS.K and a write-out one STS.K, and each slot's constants are
// decoded once for all K groups.
template <int K>
__device__ __forceinline__ void ldsK(uint32_t addr, uint32_t (&v)[K]) {
  if (K == 1) {
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v[0]) : "r"(addr));
  } else if (K == 2) {
    asm volatile("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(v[0]), "=r"(v[1]) : "r"(addr));
  } else {
    asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]) : "r"(addr));
  }
}
template <int K>
__device__ __forceinline__ void lds_leaf(uint32_t s_base, uint32_t off, uint32_t (&v)[K]) {
  if (K == 1) v[0] = *reinterpret_cast<const uint32_t*>(reinterpret_cast<const char*>(g_smem) + off);
  else ldsK<K>(s_base + K * off, v);
}
template <int K>
__device__ __forceinline__ void stsK(uint32_t addr, const uint32_t (&v)[K]) {
  if (K == 1) {
    asm volatile("st.shared.u32 [%0], %1;" ::"r"(addr), "r"(v[0]) : "memory");
  } else if (K == 2) {
    asm volatile("st.shared.v2.u32 [%0], {%1, %2};" ::"r"(addr), "r"(v[0]), "r"(v[1]) : "memory");
  } else {
    asm volatile("st.shared.v4.u32 [%0], {%1, %2, %3, %4};" ::"r"(addr), "r"(v[0]), "r"(v[1]), "r"(v[2]),
                 "r"(v[3]) : "memory");
  }
}
// bit b of a packed constant word as a full mask
__device__ __forceinline__ uint32_t cmask(uint32_t c, uint32_t b) { return (uint32_t)((int32_t)(c << (31u - b)) >> 31); }
template <int K>
__device__ __forceinline__ void kslot(uint32_t (&o)[K], const uint32_t (&A)[K], const uint32_t (&B)[K], uint32_t xa,
                                      uint32_t xb, uint32_t ob, uint32_t b) {
  const uint32_t XA = cmask(xa, b), XB = cmask(xb, b), OB = cmask(ob, b);
#pragma unroll
  for (int j = 0; j < K; j++) o[j] = (A[j] ^ XA) & ((B[j] ^ XB) | OB);
}
// levels 1-5: byte-spread constants (gem_isa.h); b is a compile-time slot bit,
// so the shift is shared by 4 slots and the mask is one PRMT sign-replicate
__device__ __forceinline__ uint32_t pmask(uint32_t c, uint32_t b) {
  uint32_t r;
  asm("prmt.b32 %0, %1, 0, %2;" : "=r"(r) : "r"(c << (b >> 2)), "r"(0x8888u + (b & 3u) * 0x1111u));
  return r;
}
template <int K>
__device__ __forceinline__ void kslotp(uint32_t (&o)[K], const uint32_t (&A)[K], const uint32_t (&B)[K], uint32_t xa,
                                       uint32_t xb, uint32_t ob, uint32_t b) {
  const uint32_t XA = pmask(xa, b), XB = pmask(xb, b), OB = pmask(ob, b);
#pragma unroll
  for (int j = 0; j < K; j++) o[j] = (A[j] ^ XA) & ((B[j] ^ XB) | OB);
}
template <int K>
__device__ __forceinline__ void lane_woK(uint32_t s_base, uint32_t mask, uint32_t base, uint32_t b,
                                         const uint32_t (&v)[K]) {
  if ((mask >> b) & 1u) stsK<K>(s_base + 4u * K * (base + __popc(mask & ((1u << b) - 1u))), v);
}

// Rows a3-a5 of one layer for the K groups of a work item.  topv[warp][K].
template <int K>
__device__ __forceinline__ void exec_lane_layer(const LaneRegs& R, uint32_t s_base, uint32_t* topv, uint32_t bid) {
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const bool uses_top = (R.flags & GEM_LF_USES_TOP) != 0;
  if ((R.flags >> warp) & 1u) {
    const uint32_t xa = R.lc.x, xb = R.lc.y, ob = R.lc.z, mask = R.lc.w;
    const uint32_t q8[4][4] = {{R.e[0].x, R.e[0].y, R.e[0].z, R.e[0].w}, {R.e[1].x, R.e[1].y, R.e[1].z, R.e[1].w},
                               {R.e[2].x, R.e[2].y, R.e[2].z, R.e[2].w}, {R.e[3].x, R.e[3].y, R.e[3].z, R.e[3].w}};
    // leaf i (0..31) = u16 byte offset (lane word * 4): entry 8g+2k in the low
    // half of q8[g][k], +1 in the high half; with K interleaved groups the
    // word's address is K * offset, for K = 1 a plain shared load off the base
    // pointer (LDS [R + UR]: one extract per leaf, no address arithmetic)
    auto leaf = [&](uint32_t i) -> uint32_t {
      const uint32_t q = q8[i >> 3][(i & 7) >> 1];
      return (i & 1) ? (q >> 16) : (q & 0xFFFFu);
    };
    // written slots go to consecutive lane words (slot-bit order) from R.base
    uint32_t wp = s_base + 4u * K * (R.base & 0xFFFFu);   // level-1 run
    uint32_t r1[16][K];
#pragma unroll
    for (uint32_t q = 0; q < 16; q++) {          // level 1: A = leaf q, B = leaf q+16
      uint32_t a[K], b[K];
      lds_leaf<K>(s_base, leaf(q), a);
      lds_leaf<K>(s_base, leaf(q + 16), b);
      kslotp<K>(r1[q], a, b, xa, xb, ob, q);
      if (mask & (1u << q)) { stsK<K>(wp, r1[q]); wp += 4u * K; }
    }
    uint32_t r2[8][K], r3[4][K], r4[2][K], x[K];
    wp = s_base + 4u * K * (R.base >> 16);                // levels 2-5 run
#pragma unroll
    for (uint32_t q = 0; q < 8; q++) {
      kslotp<K>(r2[q], r1[q], r1[q + 8], xa, xb, ob, 16 + q);
      if (mask & (1u << (16 + q))) { stsK<K>(wp, r2[q]); wp += 4u * K; }
    }
#pragma unroll
    for (uint32_t q = 0; q < 4; q++) {
      kslotp<K>(r3[q], r2[q], r2[q + 4], xa, xb, ob, 24 + q);
      if (mask & (1u << (24 + q))) { stsK<K>(wp, r3[q]); wp += 4u * K; }
    }
#pragma unroll
    for (uint32_t q = 0; q < 2; q++) {
      kslotp<K>(r4[q], r3[q], r3[q + 2], xa, xb, ob, 28 + q);
      if (mask & (1u << (28 + q))) { stsK<K>(wp, r4[q]); wp += 4u * K; }
    }
    kslotp<K>(x, r4[0], r4[1], xa, xb, ob, 30);
    if (mask & (1u << 30)) stsK<K>(wp, x);
    // levels 6-10 across the warp: slot q of a level lives in lane q
    const uint32_t wxa = R.wc.x, wxb = R.wc.y, wob = R.wc.z, wmask = R.wc.w;
    const uint32_t offs[5] = {0, 16, 24, 28, 30};
#pragma unroll
    for (uint32_t k = 0; k < 5; k++) {
      const uint32_t half = 16u >> k;
      uint32_t y[K];
#pragma unroll
      for (int j = 0; j < K; j++) y[j] = __shfl_down_sync(0xFFFFFFFFu, x[j], half);
      const uint32_t b = offs[k] + (lane & (half - 1u));
      kslot<K>(x, x, y, wxa, wxb, wob, b);
      if (lane < half) lane_woK<K>(s_base, wmask, R.wbase, b, x);
    }
    if (uses_top && lane == 0) {
#pragma unroll
      for (int j = 0; j < K; j++) topv[warp * K + j] = x[j];
    }
  } else if (uses_top && lane == 0) {
#pragma unroll
    for (int j = 0; j < K; j++) topv[warp * K + j] = 0u;
  }
  // levels 11-13: warps 1-7 arrive on named barrier `bid`; warp 0 folds in
  // top_lane_layer after loading the next layer's records
  if (uses_top && warp != 0) asm volatile("bar.arrive %0, %1;" ::"r"(bid), "r"(GEM_THREADS) : "memory");
}

// Levels 11-13 (warp 0): wait for the 8 warp words on named barrier `bid`;
// lanes 0-7 hold them and three shuffle levels fold them.
template <int K>
__device__ __forceinline__ void top_lane_layer(uint32_t topc, uint32_t topwo, uint32_t s_base, const uint32_t* topv,
                                               uint32_t bid) {
  asm volatile("bar.sync %0, %1;" ::"r"(bid), "r"(GEM_THREADS) : "memory");
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t xa = topc & 0xFFu, xb = (topc >> 8) & 0xFFu, ob = (topc >> 16) & 0xFFu;
  const uint32_t tm = topwo & 0x7Fu, tb = topwo >> 8;
  uint32_t x[K], y[K];
#pragma unroll
  for (int j = 0; j < K; j++) x[j] = topv[(lane & 7u) * K + j];
#pragma unroll
  for (int j = 0; j < K; j++) y[j] = __shfl_down_sync(0xFFFFFFFFu, x[j], 4);
  kslot<K>(x, x, y, xa, xb, ob, lane & 3u);                 // level 11: slots 0-3
  if (lane < 4) lane_woK<K>(s_base, tm, tb, lane, x);
#pragma unroll
  for (int j = 0; j < K; j++) y[j] = __shfl_down_sync(0xFFFFFFFFu, x[j], 2);
  kslot<K>(x, x, y, xa, xb, ob, 4u + (lane & 1u));          // level 12: slots 4-5
  if (lane < 2) lane_woK<K>(s_base, tm, tb, 4u + lane, x);
#pragma unroll
  for (int j = 0; j < K; j++) y[j] = __shfl_down_sync(0xFFFFFFFFu, x[j], 1);
  kslot<K>(x, x, y, xa, xb, ob, 6u);                        // level 13: slot 6
  if (lane == 0) lane_woK<K>(s_base, tm, tb, 6u, x);
}

// ---- a2 in lane mode: input ports of an item's groups (once per cycle).
// Entry k (one u32 gid per entry) goes to lane word k + 1.  A thread takes 4
// consecutive entries per uint4 and up to 16 per pass: all entry loads, then
// all value loads, then the stores (two L2 round trips per pass, not per entry)
template <int K>
__device__ __forceinline__ void lane_ports(const KParams& kp, uint32_t s_base, const uint32_t* gread, uint32_t n_gread,
                                           uint32_t g0, uint32_t ng, uint32_t c, uint32_t cur) {
  const uint32_t tid = threadIdx.x;
  const LaneIdx X{kp.n_groups};
  const uint4* gr4 = reinterpret_cast<const uint4*>(gread);
  const uint32_t* bpi[K];
  const uint32_t* bq[K];
  const uint32_t* brd[K];
  const uint32_t* bcut[K];
#pragma unroll
  for (int j = 0; j < K; j++) {
    const uint32_t g = g0 + min((uint32_t)j, ng - 1u);
    bpi[j] = kp.pi_lane + X.q(kp.in_base + c, kp.pi_words * 32, 0, g);
    bq[j] = kp.q + X.q(cur, kp.q_words * 32, 0, g);
    brd[j] = kp.rd + X.q(cur, kp.n_rams * 32, 0, g);
    bcut[j] = kp.cut + X.q(0, kp.cut_words * 32, 0, g);
  }
  constexpr uint32_t NU = K >= 4 ? 1u : 4u / K;   // uint4 entry groups per thread and pass (K * 4 * NU loads in flight)
  for (uint32_t kb = 0; kb < n_gread; kb += 4 * NU * GEM_THREADS) {
    uint4 e[NU];
#pragma unroll
    for (uint32_t u = 0; u < NU; u++) {
      const uint32_t q4 = kb / 4 + u * GEM_THREADS + tid;
      e[u] = 4 * q4 < n_gread ? __ldg(gr4 + q4) : make_uint4(0, 0, 0, 0);
    }
    // the K groups' values of the same entries are loaded together (K * 16 in flight)
    uint32_t v[K][4 * NU];
#pragma unroll
    for (uint32_t u = 0; u < NU; u++) {
      const uint32_t ev[4] = {e[u].x, e[u].y, e[u].z, e[u].w};
      const uint32_t k4 = kb + 4 * (u * GEM_THREADS + tid);
#pragma unroll
      for (uint32_t h = 0; h < 4; h++) {
        const uint32_t reg = ev[h] >> 24, b = ev[h] & 0xFFFFFFu;
        const bool ok = k4 + h < n_gread;
#pragma unroll
        for (int j = 0; j < K; j++) {
          const uint32_t* base = reg == GEM_R_PI ? bpi[j] : reg == GEM_R_Q ? bq[j] : reg == GEM_R_RD ? brd[j] : bcut[j];
          v[j][4 * u + h] = ok ? __ldcg(base + (size_t)b * X.G) : 0u;
        }
      }
    }
#pragma unroll
    for (uint32_t u = 0; u < NU; u++) {
      const uint32_t k4 = kb + 4 * (u * GEM_THREADS + tid);
#pragma unroll
      for (uint32_t h = 0; h < 4; h++)
        if (k4 + h < n_gread) {
          uint32_t w[K];
#pragma unroll
          for (int j = 0; j < K; j++) w[j] = v[j][4 * u + h];
          stsK<K>(s_base + 4u * K * (k4 + h + 1), w);   // padding groups (j >= ng) are never committed
        }
    }
  }
}

// ---- a6/a7 in lane mode: endpoint commit (one lane word per endpoint bit,
// entries of 4 endpoints per thread loaded ahead, one LDS.K for all K groups)
// and the RAM blocks (one warp per RAM, lane s = stream 32g+s; read-first,
// per-bit write).
template <int K>
__device__ __forceinline__ void lane_commit(const KParams& kp, uint32_t s_base, uint32_t* ramp, const uint32_t* outs,
                                            uint32_t n_out, const uint32_t* rr, uint32_t n_ram, uint32_t g0,
                                            uint32_t ng, uint32_t c, uint32_t nxt) {
  const uint32_t tid = threadIdx.x;
  const LaneIdx X{kp.n_groups};
  // ---- a6: endpoint commit: one lane word per endpoint bit
  // entries of 4 endpoints per thread are loaded before use; one LDS.K gives
  // the source word of all K groups
  const uint2* oe = reinterpret_cast<const uint2*>(outs);
  for (uint32_t o0 = 0; o0 < n_out; o0 += 4 * GEM_THREADS) {
    uint2 e[4];
#pragma unroll
    for (uint32_t u = 0; u < 4; u++) {
      const uint32_t o = o0 + u * GEM_THREADS + tid;
      e[u] = o < n_out ? __ldg(oe + o) : make_uint2(0, 0);
    }
#pragma unroll
    for (uint32_t u = 0; u < 4; u++) {
      if (o0 + u * GEM_THREADS + tid >= n_out) continue;
      uint32_t v[K];
      ldsK<K>(s_base + 4u * K * (e[u].y & 0xFFFFu), v);
      const uint32_t inv = (e[u].y >> 31) ? 0xFFFFFFFFu : 0u;
      const uint32_t reg = e[u].x >> 24, b = e[u].x & 0xFFFFFFu;
      uint32_t* dst = reg == GEM_R_Q ? kp.q + X.q(nxt, kp.q_words * 32, b, g0)
                    : reg == GEM_R_PO ? kp.po_lane + X.q(c, kp.po_words * 32, b, g0)
                    : reg == GEM_R_CUT ? kp.cut + X.q(0, kp.cut_words * 32, b, g0) : nullptr;
      if (dst && K == 4 && ng == 4 && (X.G & 3u) == 0 && (g0 & 3u) == 0) {
        // the item's 4 groups are one 16-byte word of the group-minor layout
        __stcg(reinterpret_cast<uint4*>(dst), make_uint4(v[0] ^ inv, v[1 % K] ^ inv, v[2 % K] ^ inv, v[3 % K] ^ inv));
        continue;
      }
#pragma unroll
      for (int j = 0; j < K; j++) {
        if ((uint32_t)j >= ng) break;
        const uint32_t x = v[j] ^ inv;
        if (dst) __stcg(dst + j, x);
        else ramp[j * kp.ramp_words + b] = x;
      }
    }
  }
  // ---- a7: RAM blocks: one warp per RAM, lane s = stream 32g+s (read-first, per-bit write)
  if (n_ram) {
    __syncthreads();
    const uint32_t lane = tid & 31;
    for (uint32_t jr = tid >> 5; jr < n_ram * ng; jr += GEM_WARPS) {
      const uint32_t j = jr / n_ram, r = jr - j * n_ram, g = g0 + j;
      const uint32_t nvalid = min(32u, kp.n_streams - 32u * g);
      const uint32_t id = __ldg(rr + 4 * r);
      const uint32_t* rp = ramp + j * kp.ramp_words + r * 128;
      uint32_t ra = 0, wa = 0, wd = 0, be = 0;
#pragma unroll
      for (uint32_t k = 0; k < 13; k++) {
        ra |= ((rp[k] >> lane) & 1u) << k;
        wa |= ((rp[32 + k] >> lane) & 1u) << k;
      }
#pragma unroll 8
      for (uint32_t k = 0; k < 32; k++) {
        wd |= ((rp[64 + k] >> lane) & 1u) << k;
        be |= ((rp[96 + k] >> lane) & 1u) << k;
      }
      uint32_t old = 0;
      if (lane < nvalid) {
        uint32_t* M = kp.mem + ((size_t)(32u * g + lane) * kp.n_rams + id) * GEM_RAM_WORDS;
        old = __ldcg(M + ra);
        const uint32_t cw = __ldcg(M + wa);
        __stcg(M + wa, (cw & ~be) | (wd & be));
      }
      // transpose the 32 read words into 32 lane words
#pragma unroll 4
      for (uint32_t k = 0; k < 32; k++) {
        const uint32_t w = __ballot_sync(0xFFFFFFFFu, (old >> k) & 1u);
        if (lane == k) __stcg(kp.rd + X.q(nxt, kp.n_rams * 32, id * 32 + k, g), w);
      }
    }
  }
}

// One work item: partition p for the 32-stream groups g0 .. g0+ng-1 (ng <= K;
// groups ng..K-1 of the vectors are padding and never committed).
template <int K>
__device__ void run_lane_partition(const KParams& kp, uint32_t* S, uint32_t* ramp, uint32_t* topv, uint32_t p,
                                   uint32_t g0, uint32_t ng, uint32_t c, uint32_t cur, uint32_t nxt,
                                   unsigned long long* pacc) {
  const uint32_t tid = threadIdx.x;
  // GEM_F_PROFILE: thread 0 accumulates per-phase clocks over the CTA's items
  unsigned long long t_ph = (pacc && tid == 0) ? clock64() : 0ull;
  auto phase = [&](int k) {
    if (pacc && tid == 0) {
      const unsigned long long t = clock64();
      pacc[k] += t - t_ph;
      t_ph = t;
    }
  };
  const uint32_t s_base = smem_u32(S);
  const LaneIdx X{kp.n_groups};
  const uint32_t* gprog = kp.lprog + __ldg(kp.parts + p * GP_WORDS + GP_LANE_OFF);
  const uint4 h0 = __ldg(reinterpret_cast<const uint4*>(gprog));
  const uint4 h1 = __ldg(reinterpret_cast<const uint4*>(gprog) + 1);
  const uint4 h2 = __ldg(reinterpret_cast<const uint4*>(gprog) + 2);
  const uint32_t n_gread = h0.y, n_layers = h0.z, n_out = h0.w;
  const uint32_t n_ram = h1.x, off_gread = h1.z, off_layers = h1.w;
  const uint32_t off_out = h2.x, off_ram = h2.y;
  // layer 0's records first: independent of S, their latency overlaps the port loads
  const uint32_t* L = gprog + off_layers;
  LaneRegs R;
  if (n_layers) load_lane_first(L, R);
  if (pacc && tid == 0 && h0.x == 0u) pacc[7]++;   // (keeps the header read before the stamp)
  phase(0);
  // ---- a2: input ports (once per cycle) for the groups of the item.
  // Entry k (one u32 gid per entry) goes to lane word k + 1.  A thread takes 4
  // consecutive entries per uint4 and up to 16 per pass: all entry loads, then
  // all value loads, then the stores (two L2 round trips per pass, not per entry)
  lane_ports<K>(kp, s_base, gprog + off_gread, n_gread, g0, ng, c, cur);
  if (tid < K) S[tid] = 0u;   // lane word 0 = constant 0 for every group
  phase(1);
  __syncthreads();
  phase(2);
  for (uint32_t l = 0; l < n_layers; l++) {
    exec_lane_layer<K>(R, s_base, topv, 1);
    const bool ptop = (R.flags & GEM_LF_USES_TOP) != 0;
    const uint32_t ptopc = R.topc, ptopwo = R.topwo;
    L += R.size;
    if (l + 1 < n_layers) load_lane_next(L, R);
    if (ptop && (threadIdx.x >> 5) == 0) top_lane_layer<K>(ptopc, ptopwo, s_base, topv, 1);
    __syncthreads();
  }
  phase(3);
  lane_commit<K>(kp, s_base, ramp, gprog + off_out, n_out, gprog + off_ram, n_ram, g0, ng, c, nxt);
  __syncthreads();
  phase(4);
}

// Input ports of a compacted lane program: entry k (one u32 gid, sorted by
// global bit) -> lane word k + 1.  Thread t takes entries t, t+256, ... so a
// warp's 32 consecutive entries -- mostly consecutive bits of one lane row --
// load as one coalesced line per group, and their STS.K are conflict-free.
template <int K>
__device__ __forceinline__ void lane_ports2(const KParams& kp, uint32_t s_base, const uint32_t* gread,
                                            uint32_t n_gread, uint32_t g0, uint32_t ng, uint32_t c, uint32_t cur) {
  const uint32_t tid = threadIdx.x;
  const LaneIdx X{kp.n_groups};
  // row bases of group 0 (X[row][bit][group]); a value is row + bit * G + group
  const uint32_t* rpi = kp.pi_lane + X.q(kp.in_base + c, kp.pi_words * 32, 0, 0);
  const uint32_t* rq = kp.q + X.q(cur, kp.q_words * 32, 0, 0);
  const uint32_t* rrd = kp.rd + X.q(cur, kp.n_rams * 32, 0, 0);
  const uint32_t* rcut = kp.cut;
  // K = 4 groups of an aligned item are one 16-byte word
  const bool vec = K == 4 && ng == 4 && (X.G & 3u) == 0 && (g0 & 3u) == 0;
  constexpr uint32_t U = K >= 4 ? 8u : 8u / K;   // entries per thread per pass (U * K loads in flight)
  for (uint32_t kb = 0; kb < n_gread; kb += U * GEM_THREADS) {
    uint32_t e[U];
#pragma unroll
    for (uint32_t u = 0; u < U; u++) {
      const uint32_t k = kb + u * GEM_THREADS + tid;
      e[u] = k < n_gread ? __ldg(gread + k) : 0xFFFFFFFFu;
    }
    uint32_t v[U][K];
#pragma unroll
    for (uint32_t u = 0; u < U; u++) {
      const uint32_t reg = e[u] >> 24, b = e[u] & 0xFFFFFFu;
      const uint32_t* row = reg == GEM_R_PI ? rpi : reg == GEM_R_Q ? rq : reg == GEM_R_RD ? rrd : rcut;
      const uint32_t* a = row + (size_t)b * X.G + g0;
      if (e[u] == 0xFFFFFFFFu) {
#pragma unroll
        for (int j = 0; j < K; j++) v[u][j] = 0u;
      } else if (vec) {
        const uint4 w4 = __ldcg(reinterpret_cast<const uint4*>(a));
        v[u][0] = w4.x; v[u][1 % K] = w4.y; v[u][2 % K] = w4.z; v[u][3 % K] = w4.w;
      } else {
#pragma unroll
        for (int j = 0; j < K; j++) v[u][j] = __ldcg(a + min((uint32_t)j, ng - 1u));
      }
    }
#pragma unroll
    for (uint32_t u = 0; u < U; u++)
      if (e[u] != 0xFFFFFFFFu) stsK<K>(s_base + 4u * K * (kb + u * GEM_THREADS + tid + 1), v[u]);
  }
}

// One work item of a compacted lane program ("LAN2", gem_isa.h): ports, then
// the partition's ANDs in barrier-separated steps of <= 256*M (thread t runs
// ops (s*M + j)*256 + t, j < M, of step s on all K groups: per op two LDS.K,
// 2K LOP3, one STS.K; the M ops of a thread are independent, so their loads
// overlap), then endpoints and RAMs.  The op words stream from the
// L2-resident program into registers kPre steps ahead of their use.
template <int K, int M>
__device__ void run_lane_partition2(const KParams& kp, uint32_t* S, uint32_t* ramp, uint32_t p, uint32_t g0,
                                    uint32_t ng, uint32_t c, uint32_t cur, uint32_t nxt, unsigned long long* pacc) {
  const uint32_t tid = threadIdx.x;
  unsigned long long t_ph = (pacc && tid == 0) ? clock64() : 0ull;
  auto phase = [&](int k) {
    if (pacc && tid == 0) {
      const unsigned long long t = clock64();
      pacc[k] += t - t_ph;
      t_ph = t;
    }
  };
  const uint32_t s_base = smem_u32(S);
  const uint32_t* gprog = kp.lprog + __ldg(kp.parts + p * GP_WORDS + GP_LANE_OFF);
  const uint4 h0 = __ldg(reinterpret_cast<const uint4*>(gprog));
  const uint4 h1 = __ldg(reinterpret_cast<const uint4*>(gprog) + 1);
  const uint4 h2 = __ldg(reinterpret_cast<const uint4*>(gprog) + 2);
  const uint32_t n_gread = h0.y, n_steps = h0.z, n_out = h0.w;
  const uint32_t n_ram = h1.x, off_gread = h1.z, off_ops = h1.w;
  const uint32_t off_out = h2.x, off_ram = h2.y;
  const uint2* ops = reinterpret_cast<const uint2*>(gprog + off_ops) + tid;
  // the first steps' ops: independent of S, their latency overlaps the port loads
  constexpr uint32_t kPre = M == 1 ? 8 : 4;
  uint2 q[kPre][M];
#pragma unroll
  for (uint32_t i = 0; i < kPre; i++)
#pragma unroll
    for (int j = 0; j < M; j++)
      q[i][j] = i < n_steps ? __ldg(ops + (i * M + j) * GEM_LANE2_STEP) : make_uint2(0u, 0u);
  phase(0);
  lane_ports2<K>(kp, s_base, gprog + off_gread, n_gread, g0, ng, c, cur);
  if (tid < K) S[tid] = 0u;   // lane word 0 = constant 0 for every group
  phase(1);
  __syncthreads();
  phase(2);
  for (uint32_t s = 0; s < n_steps; s++) {
    uint2 o[M];
#pragma unroll
    for (int j = 0; j < M; j++) o[j] = q[0][j];
#pragma unroll
    for (uint32_t i = 0; i + 1 < kPre; i++)
#pragma unroll
      for (int j = 0; j < M; j++) q[i][j] = q[i + 1][j];
#pragma unroll
    for (int j = 0; j < M; j++)
      q[kPre - 1][j] = s + kPre < n_steps ? __ldg(ops + ((s + kPre) * M + j) * GEM_LANE2_STEP) : make_uint2(0u, 0u);
    uint32_t a[M][K], b[M][K];
#pragma unroll
    for (int j = 0; j < M; j++)
      if (o[j].y) {
        ldsK<K>(s_base + 4u * K * (o[j].x & 0x3FFFu), a[j]);
        ldsK<K>(s_base + 4u * K * ((o[j].x >> 16) & 0x3FFFu), b[j]);
      }
#pragma unroll
    for (int j = 0; j < M; j++)
      if (o[j].y) {
        const uint32_t ia = (uint32_t)((int32_t)(o[j].x << 17) >> 31), ib = (uint32_t)((int32_t)(o[j].x << 1) >> 31);
        uint32_t r[K];
#pragma unroll
        for (int g = 0; g < K; g++) r[g] = (a[j][g] ^ ia) & (b[j][g] ^ ib);
        stsK<K>(s_base + 4u * K * o[j].y, r);
      }
    __syncthreads();
  }
  phase(3);
  lane_commit<K>(kp, s_base, ramp, gprog + off_out, n_out, gprog + off_ram, n_ram, g0, ng, c, nxt);
  __syncthreads();
  phase(4);
}

// Parity instruments in lane mode: flop digest / trace from the lane words.
__device__ void record_state_lane(const KParams& kp, uint32_t c, uint32_t buf) {
  const LaneIdx X{kp.n_groups};
  const uint32_t total = kp.n_streams * kp.q_ext_words;
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < total; i += gridDim.x * blockDim.x) {
    const uint32_t st = i / kp.q_ext_words, w = i % kp.q_ext_words, g = st >> 5, s = st & 31;
    uint32_t v = 0;
    for (uint32_t b = 0; b < 32; b++) {
      const uint32_t e = w * 32 + b;
      if (e >= kp.n_flops) break;
      const uint32_t in = __ldg(kp.q_int_of_ext + e);
      v |= ((__ldcg(kp.q + X.q(buf, kp.q_words * 32, in, g)) >> s) & 1u) << b;
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

template <int K, bool V2, int M>
__global__ void __launch_bounds__(GEM_THREADS, (V2 && K <= 2) ? 4 : 2) gem_lane_kernel(const KParams kp) {
  extern __shared__ __align__(16) uint32_t smem[];
  // layout: S[lane_words][K] | ramp[K][ramp_words] | topv[16][K]  (no program ring:
  // records are loaded from global memory into registers one layer ahead)
  uint32_t* S = smem;                                   // [lane word][group] interleaved
  uint32_t* ramp = S + kp.group * kp.state_words;       // [group][ramp_words]
  uint32_t* topv = ramp + kp.group * kp.ramp_words;     // [group][16]
  const uint32_t tid = threadIdx.x;
  const uint32_t G = gridDim.x, B = blockIdx.x;
  auto wl_begin = [&](uint32_t s) { return __ldg(kp.wl_off + s * (G + 1) + B); };
  auto wl_end = [&](uint32_t s) { return __ldg(kp.wl_off + s * (G + 1) + B + 1); };
  for (uint32_t k = tid; k < 16 * kp.group; k += GEM_THREADS) topv[k] = 0u;
  __syncthreads();
  const bool dyn = kp.dyn_units != nullptr;
  __shared__ uint32_t s_next[2];   // dynamic mode: next unit (double-buffered by unit parity)
  unsigned long long bar_target = 0;
  const bool instr = (kp.flags & (GEM_F_TRACE_STATE | GEM_F_DIGEST)) != 0;
  __shared__ unsigned long long pacc[8];   // GEM_F_PROFILE phase sums (thread 0)
  for (uint32_t c = 0; c < kp.ncycles; c++) {
    const uint64_t t = kp.t0 + c;
    const uint32_t cur = (uint32_t)(t & 1u), nxt = cur ^ 1u;
    const bool prof_on = kp.prof && c < kp.prof_cycles;
    if (prof_on && threadIdx.x == 0)
      for (int k = 0; k < 8; k++) pacc[k] = 0ull;
    PROF(0);
    if (instr && c > 0) record_state_lane(kp, c - 1, cur);
    if (dyn) {
      // counter of cycle c+1 was last used in cycle c-1 (all CTAs are past its barrier)
      if (B == 0 && tid == 0) atomicExch(kp.dyn_ctr + ((c + 1) & 1u), 0u);
      uint32_t u = B, par = 0;
      while (u < kp.n_units) {
        if (tid == 0) s_next[par] = atomicAdd(kp.dyn_ctr + (c & 1u), 1u) + G;
        const uint4 U = __ldg(&kp.dyn_units[u]);
        for (uint32_t r = 0; r < U.z; r++) {
          const uint32_t g0 = (U.y >> 5) + r * K;
          if (V2)
            run_lane_partition2<K, M>(kp, S, ramp, U.x, g0, min((uint32_t)K, kp.n_groups - g0), c, cur, nxt,
                                      prof_on ? pacc : nullptr);
          else
            run_lane_partition<K>(kp, S, ramp, topv, U.x, g0, min((uint32_t)K, kp.n_groups - g0), c, cur, nxt,
                                  prof_on ? pacc : nullptr);
        }
        u = s_next[par];   // written before the item's first barrier
        par ^= 1u;
      }
      PROF(4);
      grid_sync(kp, bar_target);
    } else {
      for (uint32_t s = 0; s < kp.n_stages; s++) {
        const uint32_t kb = wl_begin(s), ke = wl_end(s);
        for (uint32_t k = kb; k < ke; k++) {
          const uint2 it = __ldg(&kp.wl_items[k]);
          const uint32_t g0 = it.y >> 5;
          if (V2)
            run_lane_partition2<K, M>(kp, S, ramp, it.x, g0, min((uint32_t)K, kp.n_groups - g0), c, cur, nxt,
                                      prof_on ? pacc : nullptr);
          else
            run_lane_partition<K>(kp, S, ramp, topv, it.x, g0, min((uint32_t)K, kp.n_groups - g0), c, cur, nxt,
                                  prof_on ? pacc : nullptr);
        }
        if (s == 0) PROF(4);
        grid_sync(kp, bar_target);
      }
    }
    PROF(5);
    if (prof_on && threadIdx.x == 0)
      for (int k = 0; k < 5; k++) kp.prof[((size_t)c * gridDim.x + blockIdx.x) * GEM_PROF_SLOTS + 11 + k] = pacc[k];
  }
  if (instr) record_state_lane(kp, kp.ncycles - 1, (uint32_t)((kp.t0 + kp.ncycles) & 1u));
}

// ---- 32x32 bit transposes between per-stream words and lane words (one warp per tile)
// stream-major in[stream][row_stride...]: word w of stream s at in[s * s_stride + row * r_stride + w]
__global__ void to_lanes_kernel(const uint32_t* __restrict__ in, uint32_t* __restrict__ out, uint32_t n_streams,
                                uint32_t rows, uint32_t words, uint64_t s_stride, uint64_t r_stride,
                                uint32_t n_groups, uint64_t out_row_base) {
  // out[out_row_base + row][w*32 + k][g] = bit k of word w, lane s of group g
  const uint32_t lane = threadIdx.x & 31;
  const uint64_t warps = (uint64_t)rows * n_groups * words;
  for (uint64_t wi = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; wi < warps;
       wi += ((uint64_t)gridDim.x * blockDim.x) >> 5) {
    const uint32_t w = (uint32_t)(wi % words);
    const uint32_t g = (uint32_t)((wi / words) % n_groups);
    const uint64_t row = wi / ((uint64_t)words * n_groups);
    const uint32_t st = g * 32 + lane;
    const uint32_t x = st < n_streams ? in[st * s_stride + row * r_stride + w] : 0u;
    uint32_t mine = 0;
#pragma unroll
    for (uint32_t k = 0; k < 32; k++) {
      const uint32_t b = __ballot_sync(0xFFFFFFFFu, (x >> k) & 1u);
      if (lane == k) mine = b;
    }
    out[((out_row_base + row) * words * 32 + w * 32 + lane) * n_groups + g] = mine;   // X[row][bit][group]
  }
}

__global__ void from_lanes_kernel(const uint32_t* __restrict__ in, uint32_t* __restrict__ out, uint32_t n_streams,
                                  uint32_t rows, uint32_t words, uint64_t s_stride, uint64_t r_stride,
                                  uint32_t n_groups) {
  // inverse of to_lanes_kernel (row base 0)
  const uint32_t lane = threadIdx.x & 31;
  const uint64_t warps = (uint64_t)rows * n_groups * words;
  for (uint64_t wi = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; wi < warps;
       wi += ((uint64_t)gridDim.x * blockDim.x) >> 5) {
    const uint32_t w = (uint32_t)(wi % words);
    const uint32_t g = (uint32_t)((wi / words) % n_groups);
    const uint64_t row = wi / ((uint64_t)words * n_groups);
    const uint32_t y = in[(row * words * 32 + w * 32 + lane) * n_groups + g];   // X[row][bit][group]
    uint32_t mine = 0;
#pragma unroll
    for (uint32_t s = 0; s < 32; s++) {
      const uint32_t b = __ballot_sync(0xFFFFFFFFu, (y >> s) & 1u);
      if (lane == s) mine = b;
    }
    const uint32_t st = g * 32 + lane;
    if (st < n_streams) out[st * s_stride + row * r_stride + w] = mine;
  }
}
