// Micro-benchmark: variants of the word-mode step loop (gem_words.cuh), 1 CTA
// of 256 threads per SM, single stream, NSTEPS steps of `n` ops (n <= 256, one
// op per thread), op words resident in shared memory.  clk per step on CTA 0.
//   V0  op LDS after the barrier (ubench_steps.cu baseline)
//   V1  op words of step s+1 loaded before the barrier of step s
//   V2  V1 + per-step op count from a shared step table + `if (tid < n)`
//   V3  V2 with the next step's count loaded one step ahead
//   V4  V3 + the loop body as in gem_words.cuh (round switch)
// Build/run: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/us2 scripts/ubench_steps2.cu && /tmp/us2
#include <cstdint>
#include <cstdio>
#include <vector>
#include <random>
#include <algorithm>

#define NT 256
#define NW 4096
#define NSTEPS 64

__device__ __forceinline__ uint32_t lds(uint32_t a) {
  uint32_t v;
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ void sts(uint32_t a, uint32_t v) {
  asm volatile("st.shared.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ uint2 lds64(uint32_t addr) {
  uint2 r;
  asm volatile("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(r.x), "=r"(r.y) : "r"(addr));
  return r;
}

template <int V>
__global__ void __launch_bounds__(NT, 1) k(const uint2* __restrict__ ops, const uint32_t* __restrict__ cnt,
                                           unsigned long long* out, int reps) {
  extern __shared__ __align__(16) uint32_t sm[];
  uint32_t* S = sm;
  uint2* O = reinterpret_cast<uint2*>(sm + NW);
  uint32_t* C = sm + NW + 2 * (NSTEPS + 1) * NT;
  const uint32_t tid = threadIdx.x;
  for (uint32_t i = tid; i < NW; i += NT) S[i] = i * 2654435761u;
  for (uint32_t i = tid; i < NSTEPS * NT; i += NT) O[i] = ops[i];
  for (uint32_t i = tid; i < 2 * (NSTEPS + 2); i += NT) C[i] = cnt[i];
  __syncthreads();
  const uint32_t sb = (uint32_t)__cvta_generic_to_shared(S);
  const uint32_t ob = (uint32_t)__cvta_generic_to_shared(O) + 8 * tid;
  const uint32_t cb = (uint32_t)__cvta_generic_to_shared(C);
  unsigned long long t0 = 0;
  for (int r = 0; r < reps; r++) {
    if (r == 2) t0 = clock64();
    if (V == 0) {
      for (int s = 0; s < NSTEPS; s++) {
        const uint2 o = lds64(ob + 8 * NT * s);
        const uint32_t a = lds(sb + (o.x & 0xFFFCu)), b = lds(sb + ((o.x >> 16) & 0xFFFCu));
        sts(sb + o.y, (a ^ o.x) & (b ^ (o.x >> 16)));
        __syncthreads();
      }
    } else if (V == 1) {
      uint2 o = lds64(ob);
      for (int s = 0; s < NSTEPS; s++) {
        const uint32_t a = lds(sb + (o.x & 0xFFFCu)), b = lds(sb + ((o.x >> 16) & 0xFFFCu));
        sts(sb + o.y, (a ^ o.x) & (b ^ (o.x >> 16)));
        if (s + 1 < NSTEPS) o = lds64(ob + 8 * NT * (s + 1));
        __syncthreads();
      }
    } else if (V == 2) {
      uint32_t n = lds(cb);
      uint2 o = make_uint2(0, 0);
      if (tid < n) o = lds64(ob);
      for (int s = 0; s < NSTEPS; s++) {
        if (tid < n) {
          const uint32_t a = lds(sb + (o.x & 0xFFFCu)), b = lds(sb + ((o.x >> 16) & 0xFFFCu));
          sts(sb + o.y, (a ^ o.x) & (b ^ (o.x >> 16)));
        }
        n = lds(cb + 4 * (s + 1));
        if (tid < n) o = lds64(ob + 8 * NT * (s + 1));
        __syncthreads();
      }
    } else if (V == 3) {
      uint32_t n = lds(cb), n1 = lds(cb + 4);
      uint2 o = make_uint2(0, 0);
      if (tid < n) o = lds64(ob);
      for (int s = 0; s < NSTEPS; s++) {
        const uint32_t n2 = lds(cb + 4 * (s + 2));
        if (tid < n) {
          const uint32_t a = lds(sb + (o.x & 0xFFFCu)), b = lds(sb + ((o.x >> 16) & 0xFFFCu));
          sts(sb + o.y, (a ^ o.x) & (b ^ (o.x >> 16)));
        }
        if (tid < n1) o = lds64(ob + 8 * NT * (s + 1));
        n = n1;
        n1 = n2;
        __syncthreads();
      }
    } else if (V == 5) {
      // V5: the step loop of gem_words.cuh (round switch, load_ops lambda)
      const uint32_t* stp = C;   // cumulative starts built on the host for V5
      const uint32_t o_base = ob;
      uint2 o[4] = {make_uint2(0u, 0u), make_uint2(0u, 0u), make_uint2(0u, 0u), make_uint2(0u, 0u)};
      auto load_ops = [&](uint32_t b0, uint32_t m) {
        const uint32_t a = o_base + 8u * b0;
        if (tid < m) o[0] = lds64(a);
        if (m > NT) {
          if (tid + NT < m) o[1] = lds64(a + 8u * NT);
          if (m > 2 * NT) {
            if (tid + 2 * NT < m) o[2] = lds64(a + 16u * NT);
            if (m > 3 * NT && tid + 3 * NT < m) o[3] = lds64(a + 24u * NT);
          }
        }
      };
      const uint32_t n_steps = NSTEPS;
      uint32_t e0 = 0, e1 = stp[1];
      load_ops(0u, e1);
      for (uint32_t s = 0; s < n_steps; s++) {
        const uint32_t e2 = s + 2 <= n_steps ? stp[s + 2] : e1;
        const uint32_t n = e1 - e0;
        if (n <= NT) {
          if (tid < n) {
            const uint32_t a = lds(sb + (o[0].x & 0xFFFCu)), b = lds(sb + ((o[0].x >> 16) & 0xFFFCu));
            sts(sb + o[0].y, (a ^ o[0].x) & (b ^ (o[0].x >> 16)));
          }
        } else {
          uint32_t a[4], b[4];
          for (int r = 0; r < 4; r++) { a[r] = lds(sb + (o[r].x & 0xFFFCu)); b[r] = lds(sb + ((o[r].x >> 16) & 0xFFFCu)); }
          for (int r = 0; r < 4; r++) sts(sb + o[r].y, (a[r] ^ o[r].x) & (b[r] ^ (o[r].x >> 16)));
        }
        load_ops(e1, e2 - e1);
        e0 = e1;
        e1 = e2;
        __syncthreads();
      }
    } else if (V == 8) {
      // V5: the step loop of gem_words.cuh (round switch, load_ops lambda)
      const uint32_t* stp = C;   // cumulative starts built on the host for V5
      const uint32_t o_base = ob;
      uint2 o[4] = {make_uint2(0u, 0u), make_uint2(0u, 0u), make_uint2(0u, 0u), make_uint2(0u, 0u)};
      auto load_ops = [&](uint32_t b0, uint32_t m) {
        const uint32_t a = o_base + 8u * b0;
        if (tid < m) o[0] = lds64(a);
        if (m > NT) {
          if (tid + NT < m) o[1] = lds64(a + 8u * NT);
          if (m > 2 * NT) {
            if (tid + 2 * NT < m) o[2] = lds64(a + 16u * NT);
            if (m > 3 * NT && tid + 3 * NT < m) o[3] = lds64(a + 24u * NT);
          }
        }
      };
      const uint32_t n_steps = NSTEPS;
      uint32_t e0 = 0, e1 = stp[1];
      load_ops(0u, e1);
      for (uint32_t s = 0; s < n_steps; s++) {
        const uint32_t e2 = s + 2 <= n_steps ? stp[s + 2] : e1;
        const uint32_t n = e1 - e0;
        if (n <= NT) {
          if (tid < n) {
            const uint32_t a = lds(sb + (o[0].x & 0xFFFCu)), b = lds(sb + ((o[0].x >> 16) & 0xFFFCu));
            sts(sb + o[0].y, (a ^ o[0].x) & (b ^ (o[0].x >> 16)));
          }
        }
        load_ops(e1, e2 - e1);
        e0 = e1;
        e1 = e2;
        __syncthreads();
      }
    } else if (V == 9) {
      // V5: the step loop of gem_words.cuh (round switch, load_ops lambda)
      const uint32_t* stp = C;   // cumulative starts built on the host for V5
      const uint32_t o_base = ob;
      uint2 o[4] = {make_uint2(0u, 0u), make_uint2(0u, 0u), make_uint2(0u, 0u), make_uint2(0u, 0u)};
      auto load_ops = [&](uint32_t b0, uint32_t m) {
        const uint32_t a = o_base + 8u * b0;
        if (tid < m) o[0] = lds64(a);
      };
      const uint32_t n_steps = NSTEPS;
      uint32_t e0 = 0, e1 = stp[1];
      load_ops(0u, e1);
      for (uint32_t s = 0; s < n_steps; s++) {
        const uint32_t e2 = s + 2 <= n_steps ? stp[s + 2] : e1;
        const uint32_t n = e1 - e0;
        if (n <= NT) {
          if (tid < n) {
            const uint32_t a = lds(sb + (o[0].x & 0xFFFCu)), b = lds(sb + ((o[0].x >> 16) & 0xFFFCu));
            sts(sb + o[0].y, (a ^ o[0].x) & (b ^ (o[0].x >> 16)));
          }
        } else {
          uint32_t a[4], b[4];
          for (int r = 0; r < 4; r++) { a[r] = lds(sb + (o[r].x & 0xFFFCu)); b[r] = lds(sb + ((o[r].x >> 16) & 0xFFFCu)); }
          for (int r = 0; r < 4; r++) sts(sb + o[r].y, (a[r] ^ o[r].x) & (b[r] ^ (o[r].x >> 16)));
        }
        load_ops(e1, e2 - e1);
        e0 = e1;
        e1 = e2;
        __syncthreads();
      }
    } else if (V == 10) {
      // V5: the step loop of gem_words.cuh (round switch, load_ops lambda)
      const uint32_t* stp = C;   // cumulative starts built on the host for V5
      const uint32_t o_base = ob;
      uint2 o[4] = {make_uint2(0u, 0u), make_uint2(0u, 0u), make_uint2(0u, 0u), make_uint2(0u, 0u)};
      auto load_ops = [&](uint32_t b0, uint32_t m) {
        const uint32_t a = o_base + 8u * b0;
        if (tid < m) o[0] = lds64(a);
      };
      const uint32_t n_steps = NSTEPS;
      uint32_t e0 = 0, e1 = stp[1];
      load_ops(0u, e1);
      for (uint32_t s = 0; s < n_steps; s++) {
        const uint32_t e2 = s + 2 <= n_steps ? stp[s + 2] : e1;
        const uint32_t n = e1 - e0;
        if (n <= NT) {
          if (tid < n) {
            const uint32_t a = lds(sb + (o[0].x & 0xFFFCu)), b = lds(sb + ((o[0].x >> 16) & 0xFFFCu));
            sts(sb + o[0].y, (a ^ o[0].x) & (b ^ (o[0].x >> 16)));
          }
        }
        load_ops(e1, e2 - e1);
        e0 = e1;
        e1 = e2;
        __syncthreads();
      }
    } else if (V == 6) {
      // V6: bounds two steps ahead, next step's ops loaded at the START of the step
      const uint32_t* stp = C;
      const uint32_t o_base = ob;
      uint2 o[4] = {make_uint2(0u, 0u), make_uint2(0u, 0u), make_uint2(0u, 0u), make_uint2(0u, 0u)};
      uint2 q[4] = {make_uint2(0u, 0u), make_uint2(0u, 0u), make_uint2(0u, 0u), make_uint2(0u, 0u)};
      auto load_ops = [&](uint2 (&r)[4], uint32_t b0, uint32_t m) {
        const uint32_t a = o_base + 8u * b0;
        if (tid < m) r[0] = lds64(a);
        if (m > NT) {
          if (tid + NT < m) r[1] = lds64(a + 8u * NT);
          if (m > 2 * NT) {
            if (tid + 2 * NT < m) r[2] = lds64(a + 16u * NT);
            if (m > 3 * NT && tid + 3 * NT < m) r[3] = lds64(a + 24u * NT);
          }
        }
      };
      const uint32_t n_steps = NSTEPS;
      uint32_t e0 = 0, e1 = stp[1], e2 = stp[2];
      load_ops(o, 0u, e1);
      for (uint32_t s = 0; s < n_steps; s++) {
        const uint32_t e3 = s + 3 <= n_steps ? stp[s + 3] : e2;
        load_ops(q, e1, e2 - e1);
        const uint32_t n = e1 - e0;
        if (n <= NT) {
          if (tid < n) {
            const uint32_t a = lds(sb + (o[0].x & 0xFFFCu)), b = lds(sb + ((o[0].x >> 16) & 0xFFFCu));
            sts(sb + o[0].y, (a ^ o[0].x) & (b ^ (o[0].x >> 16)));
          }
        } else {
          uint32_t a[4], b[4];
          for (int r = 0; r < 4; r++) { a[r] = lds(sb + (o[r].x & 0xFFFCu)); b[r] = lds(sb + ((o[r].x >> 16) & 0xFFFCu)); }
          for (int r = 0; r < 4; r++) sts(sb + o[r].y, (a[r] ^ o[r].x) & (b[r] ^ (o[r].x >> 16)));
        }
#pragma unroll
        for (int r = 0; r < 4; r++) o[r] = q[r];
        e0 = e1;
        e1 = e2;
        e2 = e3;
        __syncthreads();
      }
    } else if (V == 11) {
      // V6: bounds two steps ahead, next step's ops loaded at the START of the step
      const uint32_t* stp = C;
      const uint32_t o_base = ob;
      uint2 o[4] = {make_uint2(0u, 0u), make_uint2(0u, 0u), make_uint2(0u, 0u), make_uint2(0u, 0u)};
      uint2 q[4] = {make_uint2(0u, 0u), make_uint2(0u, 0u), make_uint2(0u, 0u), make_uint2(0u, 0u)};
      auto load_ops = [&](uint2 (&r)[4], uint32_t b0, uint32_t m) {
        const uint32_t a = o_base + 8u * b0;
        if (tid < m) r[0] = lds64(a);
      };
      const uint32_t n_steps = NSTEPS;
      uint32_t e0 = 0, e1 = stp[1], e2 = stp[2];
      load_ops(o, 0u, e1);
      for (uint32_t s = 0; s < n_steps; s++) {
        const uint32_t e3 = s + 3 <= n_steps ? stp[s + 3] : e2;
        load_ops(q, e1, e2 - e1);
        const uint32_t n = e1 - e0;
        if (n <= NT) {
          if (tid < n) {
            const uint32_t a = lds(sb + (o[0].x & 0xFFFCu)), b = lds(sb + ((o[0].x >> 16) & 0xFFFCu));
            sts(sb + o[0].y, (a ^ o[0].x) & (b ^ (o[0].x >> 16)));
          }
        }
#pragma unroll
        for (int r = 0; r < 1; r++) o[r] = q[r];
        e0 = e1;
        e1 = e2;
        e2 = e3;
        __syncthreads();
      }
    } else if (V == 12) {
      // V6: bounds two steps ahead, next step's ops loaded at the START of the step
      const uint32_t* stp = C;
      const uint32_t o_base = ob;
      uint2 o[4] = {make_uint2(0u, 0u), make_uint2(0u, 0u), make_uint2(0u, 0u), make_uint2(0u, 0u)};
      uint2 q[4] = {make_uint2(0u, 0u), make_uint2(0u, 0u), make_uint2(0u, 0u), make_uint2(0u, 0u)};
      auto load_ops = [&](uint2 (&r)[4], uint32_t b0, uint32_t m) {
        const uint32_t a = o_base + 8u * b0;
        if (tid < m) r[0] = lds64(a);
        if (m > NT && tid + NT < m) r[1] = lds64(a + 8u * NT);
      };
      const uint32_t n_steps = NSTEPS;
      uint32_t e0 = 0, e1 = stp[1], e2 = stp[2];
      load_ops(o, 0u, e1);
      for (uint32_t s = 0; s < n_steps; s++) {
        const uint32_t e3 = s + 3 <= n_steps ? stp[s + 3] : e2;
        load_ops(q, e1, e2 - e1);
        const uint32_t n = e1 - e0;
        if (n <= NT) {
          if (tid < n) {
            const uint32_t a = lds(sb + (o[0].x & 0xFFFCu)), b = lds(sb + ((o[0].x >> 16) & 0xFFFCu));
            sts(sb + o[0].y, (a ^ o[0].x) & (b ^ (o[0].x >> 16)));
          }
        } else {
          const bool ok = tid + NT < n;
          const uint32_t a0 = lds(sb + (o[0].x & 0xFFFCu)), b0 = lds(sb + ((o[0].x >> 16) & 0xFFFCu));
          uint32_t a1 = 0, b1 = 0;
          if (ok) { a1 = lds(sb + (o[1].x & 0xFFFCu)); b1 = lds(sb + ((o[1].x >> 16) & 0xFFFCu)); }
          sts(sb + o[0].y, (a0 ^ o[0].x) & (b0 ^ (o[0].x >> 16)));
          if (ok) sts(sb + o[1].y, (a1 ^ o[1].x) & (b1 ^ (o[1].x >> 16)));
        }
#pragma unroll
        for (int r = 0; r < 2; r++) o[r] = q[r];
        e0 = e1;
        e1 = e2;
        e2 = e3;
        __syncthreads();
      }
    } else if (V == 13) {
      // V13: packed step table (start | n << 16), op + operand addresses of step s+1
      // prepared during step s
      const uint32_t* tab = C;   // host: start | n << 16 per step (+ 2 padding entries)
      const uint32_t o_base = ob;
      const uint32_t n_steps = tab[NSTEPS + 1] + NSTEPS;   // runtime count
      uint32_t t0 = tab[0], t1 = tab[1];
      uint2 o = make_uint2(0u, 0u);
      if (tid < (t0 >> 16)) o = lds64(o_base + 8u * (t0 & 0xFFFFu));
      uint32_t aA = sb + (o.x & 0xFFFCu), bA = sb + ((o.x >> 16) & 0xFFFCu), xh = o.x >> 16;
      bool v = tid < (t0 >> 16);
      for (uint32_t s = 0; s < n_steps; s++) {
        const uint32_t t2 = tab[s + 2];
        uint2 q = make_uint2(0u, 0u);
        const bool vq = tid < (t1 >> 16);
        if (vq) q = lds64(o_base + 8u * (t1 & 0xFFFFu));
        if (v) {
          const uint32_t a = lds(aA), b = lds(bA);
          sts(sb + o.y, (a ^ o.x) & (b ^ xh));
        }
        o = q;
        v = vq;
        aA = sb + (o.x & 0xFFFCu);
        bA = sb + ((o.x >> 16) & 0xFFFCu);
        xh = o.x >> 16;
        t1 = t2;
        __syncthreads();
      }
    } else if (V == 16) {
      // V13: packed step table (start | n << 16), op + operand addresses of step s+1
      // prepared during step s
      const uint32_t* tab = C;   // host: start | n << 16 per step (+ 2 padding entries)
      const uint32_t o_base = ob;
      const uint32_t n_steps = tab[NSTEPS + 1] + NSTEPS;   // runtime count
      uint32_t t0 = tab[0], t1 = tab[1];
      uint2 o = make_uint2(0u, 0u);
      if (tid < (t0 >> 16)) o = lds64(o_base + 8u * (t0 & 0xFFFFu));
      uint32_t aA = sb + (o.x & 0xFFFCu), bA = sb + ((o.x >> 16) & 0xFFFCu), xh = o.x >> 16;
      bool v = tid < (t0 >> 16);
      for (uint32_t s = 0; s < n_steps; s++) {
        if (v) {
          const uint32_t a = lds(aA), b = lds(bA);
          sts(sb + o.y, (a ^ o.x) & (b ^ xh));
        }
        const uint32_t t2 = lds(cb + 4u * (s + 2));
        uint2 q = make_uint2(0u, 0u);
        const bool vq = tid < (t1 >> 16);
        if (vq) q = lds64(o_base + 8u * (t1 & 0xFFFFu));
        o = q;
        v = vq;
        aA = sb + (o.x & 0xFFFCu);
        bA = sb + ((o.x >> 16) & 0xFFFCu);
        xh = o.x >> 16;
        t1 = t2;
        __syncthreads();
      }
    } else if (V == 14) {
      // V13: packed step table (start | n << 16), op + operand addresses of step s+1
      // prepared during step s
      const uint32_t* tab = C;   // host: start | n << 16 per step (+ 2 padding entries)
      const uint32_t o_base = ob;
      const uint32_t n_steps = tab[NSTEPS + 1] + NSTEPS;   // runtime count (host writes 0 there)
      uint32_t t0 = tab[0], t1 = tab[1];
      uint2 o = make_uint2(0u, 0u);
      if (tid < (t0 >> 16)) o = lds64(o_base + 8u * (t0 & 0xFFFFu));
      uint32_t aA = sb + (o.x & 0xFFFCu), bA = sb + ((o.x >> 16) & 0xFFFCu), xh = o.x >> 16;
      bool v = tid < (t0 >> 16);
#pragma unroll 4
      for (uint32_t s = 0; s < n_steps; s++) {
        const uint32_t t2 = tab[s + 2];
        uint2 q = make_uint2(0u, 0u);
        const bool vq = tid < (t1 >> 16);
        if (vq) q = lds64(o_base + 8u * (t1 & 0xFFFFu));
        if (v) {
          const uint32_t a = lds(aA), b = lds(bA);
          sts(sb + o.y, (a ^ o.x) & (b ^ xh));
        }
        o = q;
        v = vq;
        aA = sb + (o.x & 0xFFFCu);
        bA = sb + ((o.x >> 16) & 0xFFFCu);
        xh = o.x >> 16;
        t1 = t2;
        __syncthreads();
      }
    } else if (V == 15) {
      // V13: packed step table (start | n << 16), op + operand addresses of step s+1
      // prepared during step s
      const uint32_t* tab = C;   // host: start | n << 16 per step (+ 2 padding entries)
      const uint32_t o_base = ob;
      const uint32_t n_steps = tab[NSTEPS + 1] + NSTEPS;   // runtime count
      uint32_t t0 = tab[0], t1 = tab[1];
      uint2 o = make_uint2(0u, 0u);
      if (tid < (t0 >> 16)) o = lds64(o_base + 8u * (t0 & 0xFFFFu));
      uint32_t aA = sb + (o.x & 0xFFFCu), bA = sb + ((o.x >> 16) & 0xFFFCu), xh = o.x >> 16;
      bool v = tid < (t0 >> 16);
#pragma unroll 2
      for (uint32_t s = 0; s < n_steps; s++) {
        const uint32_t t2 = tab[s + 2];
        uint2 q = make_uint2(0u, 0u);
        const bool vq = tid < (t1 >> 16);
        if (vq) q = lds64(o_base + 8u * (t1 & 0xFFFFu));
        if (v) {
          const uint32_t a = lds(aA), b = lds(bA);
          sts(sb + o.y, (a ^ o.x) & (b ^ xh));
        }
        o = q;
        v = vq;
        aA = sb + (o.x & 0xFFFCu);
        bA = sb + ((o.x >> 16) & 0xFFFCu);
        xh = o.x >> 16;
        t1 = t2;
        __syncthreads();
      }
    } else if (V == 17) {
      // V17: packed table; after the barrier: operand addresses from the op word,
      // operand loads, store; then table entry s+2 and op of s+1 (consumed after the barrier)
      const uint32_t* tab = C;
      const uint32_t o_base = ob;
      const uint32_t n_steps = tab[NSTEPS + 1] + NSTEPS;
      uint32_t t0 = tab[0], t1 = tab[1];
      uint2 o = make_uint2(0u, 0u);
      bool v = tid < (t0 >> 16);
      if (v) o = lds64(o_base + 8u * (t0 & 0xFFFFu));
      for (uint32_t s = 0; s < n_steps; s++) {
        if (v) {
          const uint32_t a = lds(sb + (o.x & 0xFFFCu)), b = lds(sb + ((o.x >> 16) & 0xFFFCu));
          sts(sb + o.y, (a ^ o.x) & (b ^ (o.x >> 16)));
        }
        const uint32_t t2 = lds(cb + 4u * (s + 2));
        v = tid < (t1 >> 16);
        if (v) o = lds64(o_base + 8u * (t1 & 0xFFFFu));
        t1 = t2;
        __syncthreads();
      }
    } else if (V == 18) {
      // V18: the WRD2 loop of gem_words.cuh (uniform 2-level form, table entries
      // {first, n1 | n2 << 16}, ops two steps ahead, S at shared address 1024)
      const uint32_t* tab = C;   // host: {first slot, n1} pairs
      const uint32_t ops_base = (uint32_t)__cvta_generic_to_shared(O);
      const uint32_t ns = NSTEPS;
      auto tabe = [&](uint32_t k) { return lds64(cb + 8u * min(k, ns)); };
      auto op_of = [&](uint2 t) -> uint3 {
        const uint32_t n1 = t.y & 0xFFFFu, n2 = t.y >> 16;
        uint3 r = make_uint3(0u, 0u, 0u);
        if (tid < n1) {
          const uint2 q = lds64(ops_base + 8u * (t.x + tid));
          r = make_uint3(q.x, 0x00010001u, q.y);
        } else if (tid < n1 + n2) {
          uint4 q;
          asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(q.x), "=r"(q.y), "=r"(q.z), "=r"(q.w)
                       : "r"(ops_base + 8u * (((t.x + n1 + 1u) & ~1u) + 2u * (tid - n1))));
          r = make_uint3(q.x, q.y, q.z);
        }
        return r;
      };
      uint2 t0 = tabe(0), t1 = tabe(1), t2 = tabe(2);
      uint3 o = op_of(t0), o1 = op_of(t1);
      for (uint32_t s = 0; s < ns; s++) {
        const uint2 t3 = tabe(s + 3);
        const uint3 o2 = op_of(t2);
        {
          const uint32_t a1 = lds(sb + (o.x & 0xFFFCu)), b1 = lds(sb + ((o.x >> 16) & 0xFFFCu));
          const uint32_t a2 = lds(sb + (o.y & 0xFFFCu)), b2 = lds(sb + ((o.y >> 16) & 0xFFFCu));
          const uint32_t u = (a1 ^ o.x) & (b1 ^ (o.x >> 16)), v = (a2 ^ o.y) & (b2 ^ (o.y >> 16));
          const uint32_t r = (u ^ o.z) & (v ^ (o.z >> 1)), d = o.z & 0xFFFCu;
          if (d) sts(sb + d, r);
        }
        o = o1;
        o1 = o2;
        t0 = t1;
        t1 = t2;
        t2 = t3;
        __syncthreads();
      }
    } else if (V == 19) {
      // V18: the WRD2 loop of gem_words.cuh (uniform 2-level form, table entries
      // {first, n1 | n2 << 16}, ops two steps ahead, S at shared address 1024)
      const uint32_t* tab = C;   // host: {first slot, n1} pairs
      const uint32_t ops_base = (uint32_t)__cvta_generic_to_shared(O);
      const uint32_t ns = NSTEPS;
      auto tabe = [&](uint32_t k) { return lds64(cb + 8u * min(k, ns)); };
      const uint32_t wlo = tid & ~31u;
      auto op_of = [&](uint2 t) -> uint3 {
        const uint32_t n1 = t.y & 0xFFFFu, n2 = t.y >> 16;
        uint3 r = make_uint3(0u, 0u, 0u);
        if (wlo >= n1 + n2) return r;   // warp-uniform: no op for this warp
        if (tid < n1) {
          const uint2 q = lds64(ops_base + 8u * (t.x + tid));
          r = make_uint3(q.x, 0x00010001u, q.y);
        } else if (tid < n1 + n2) {
          uint4 q;
          asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(q.x), "=r"(q.y), "=r"(q.z), "=r"(q.w)
                       : "r"(ops_base + 8u * (((t.x + n1 + 1u) & ~1u) + 2u * (tid - n1))));
          r = make_uint3(q.x, q.y, q.z);
        }
        return r;
      };
      uint2 t0 = tabe(0), t1 = tabe(1), t2 = tabe(2);
      uint3 o = op_of(t0), o1 = op_of(t1);
      for (uint32_t s = 0; s < ns; s++) {
        const uint2 t3 = tabe(s + 3);
        const uint3 o2 = op_of(t2);
        if (wlo < (t0.y & 0xFFFFu) + (t0.y >> 16)) {
          const uint32_t a1 = lds(sb + (o.x & 0xFFFCu)), b1 = lds(sb + ((o.x >> 16) & 0xFFFCu));
          const uint32_t a2 = lds(sb + (o.y & 0xFFFCu)), b2 = lds(sb + ((o.y >> 16) & 0xFFFCu));
          const uint32_t u = (a1 ^ o.x) & (b1 ^ (o.x >> 16)), v = (a2 ^ o.y) & (b2 ^ (o.y >> 16));
          const uint32_t r = (u ^ o.z) & (v ^ (o.z >> 1)), d = o.z & 0xFFFCu;
          if (d) sts(sb + d, r);
        }
        o = o1;
        o1 = o2;
        t0 = t1;
        t1 = t2;
        t2 = t3;
        __syncthreads();
      }
    } else if (V == 7) {
      // V7: V5 with the loop-carried bound rotated by asm-volatile moves after the stores
      const uint32_t* stp = C;
      const uint32_t o_base = ob;
      const uint32_t st_base = cb;
      uint2 o[4] = {make_uint2(0u, 0u), make_uint2(0u, 0u), make_uint2(0u, 0u), make_uint2(0u, 0u)};
      auto load_ops = [&](uint32_t b0, uint32_t m) {
        const uint32_t a = o_base + 8u * b0;
        if (tid < m) o[0] = lds64(a);
        if (m > NT) {
          if (tid + NT < m) o[1] = lds64(a + 8u * NT);
          if (m > 2 * NT) {
            if (tid + 2 * NT < m) o[2] = lds64(a + 16u * NT);
            if (m > 3 * NT && tid + 3 * NT < m) o[3] = lds64(a + 24u * NT);
          }
        }
      };
      const uint32_t n_steps = NSTEPS;
      uint32_t e0 = 0, e1 = stp[1];
      load_ops(0u, e1);
      for (uint32_t s = 0; s < n_steps; s++) {
        const uint32_t e2 = lds(st_base + 4u * min(s + 2, n_steps));
        const uint32_t n = e1 - e0;
        if (n <= NT) {
          if (tid < n) {
            const uint32_t a = lds(sb + (o[0].x & 0xFFFCu)), b = lds(sb + ((o[0].x >> 16) & 0xFFFCu));
            sts(sb + o[0].y, (a ^ o[0].x) & (b ^ (o[0].x >> 16)));
          }
        } else {
          uint32_t a[4], b[4];
          for (int r = 0; r < 4; r++) { a[r] = lds(sb + (o[r].x & 0xFFFCu)); b[r] = lds(sb + ((o[r].x >> 16) & 0xFFFCu)); }
          for (int r = 0; r < 4; r++) sts(sb + o[r].y, (a[r] ^ o[r].x) & (b[r] ^ (o[r].x >> 16)));
        }
        uint32_t e2m;
        asm volatile("mov.u32 %0, %1;" : "=r"(e2m) : "r"(e2));
        load_ops(e1, e2m - e1);
        e0 = e1;
        e1 = e2m;
        __syncthreads();
      }
    } else {
      // V4: predicated (no branch) single op, validity from the op word
      uint2 o = lds64(ob);
      for (int s = 0; s < NSTEPS; s++) {
        const uint32_t a = lds(sb + (o.x & 0xFFFCu)), b = lds(sb + ((o.x >> 16) & 0xFFFCu));
        if (o.y) sts(sb + o.y, (a ^ o.x) & (b ^ (o.x >> 16)));
        if (s + 1 < NSTEPS) o = lds64(ob + 8 * NT * (s + 1));
        __syncthreads();
      }
    }
  }
  unsigned long long t1 = clock64();
  if (tid == 0) out[blockIdx.x] = (t1 - t0) / ((unsigned long long)(reps - 2) * NSTEPS);
}

template <int V>
void run(const char* name, const uint2* d_ops, const uint32_t* d_cnt, unsigned long long* d_out, int G) {
  const size_t smem = NW * 4 + (size_t)(NSTEPS + 1) * NT * 8 + 2 * (NSTEPS + 2) * 4;
  cudaFuncSetAttribute(k<V>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  k<V><<<G, NT, smem>>>(d_ops, d_cnt, d_out, 4);
  k<V><<<G, NT, smem>>>(d_ops, d_cnt, d_out, 40);
  cudaError_t e = cudaDeviceSynchronize();
  std::vector<unsigned long long> h(G);
  cudaMemcpy(h.data(), d_out, G * 8, cudaMemcpyDeviceToHost);
  double m = 0;
  for (auto x : h) m += x;
  printf("%-52s %6.0f clk/step  (%s)\n", name, m / G, cudaGetErrorString(e));
}

int main() {
  const int G = 148;
  for (int conflict = 0; conflict < 2; conflict++)
    for (int fill : {256, 64}) {
      std::mt19937 rng(3);
      std::vector<uint2> ops((size_t)NSTEPS * NT);
      std::vector<uint32_t> cnt(2 * (NSTEPS + 2), fill);
      for (size_t i = 0; i < ops.size(); i++) {
        const uint32_t t = i % NT;
        uint32_t a = 1 + rng() % (NW - 1), b = 1 + rng() % (NW - 1);
        if (!conflict) { a = (a & ~31u) | (t & 31); b = (b & ~31u) | ((t + 7) & 31); }
        const uint32_t d = 32 * (1 + (i / NT) % 100) + (t & 31) + 32 * 100 * (t / 32 % 1);
        ops[i].x = (a * 4) | ((b * 4) << 16);
        ops[i].y = t < (uint32_t)fill ? ((d % NW) | 1) * 4 % (NW * 4) : 0;
        if (ops[i].y == 0 && t < (uint32_t)fill) ops[i].y = 4;
      }
      uint2* d_ops;
      uint32_t* d_cnt;
      unsigned long long* d_out;
      cudaMalloc(&d_ops, ops.size() * 8);
      cudaMemcpy(d_ops, ops.data(), ops.size() * 8, cudaMemcpyHostToDevice);
      cudaMalloc(&d_cnt, cnt.size() * 4);
      cudaMemcpy(d_cnt, cnt.data(), cnt.size() * 4, cudaMemcpyHostToDevice);
      cudaMalloc(&d_out, G * 8);
      printf("-- %s operands, %d ops per step\n", conflict ? "random" : "conflict-free", fill);
      run<0>("V0 op LDS after barrier", d_ops, d_cnt, d_out, G);
      run<1>("V1 op prefetched before barrier", d_ops, d_cnt, d_out, G);
      run<2>("V2 V1 + count table + if (tid < n)", d_ops, d_cnt, d_out, G);
      run<3>("V3 V2 with count 2 steps ahead", d_ops, d_cnt, d_out, G);
      run<4>("V4 V1 predicated on dst != 0", d_ops, d_cnt, d_out, G);
      {
        std::vector<uint32_t> st(NSTEPS + 2);
        for (int i = 0; i < NSTEPS + 2; i++) st[i] = std::min(i, NSTEPS) * fill;
        std::vector<uint2> packed((size_t)NSTEPS * NT);
        for (int q = 0; q < NSTEPS; q++) for (int t = 0; t < fill; t++) packed[(size_t)q * fill + t] = ops[(size_t)q * NT + t];
        cudaMemcpy(d_ops, packed.data(), packed.size() * 8, cudaMemcpyHostToDevice);
        cudaMemcpy(d_cnt, st.data(), st.size() * 4, cudaMemcpyHostToDevice);
        run<5>("V5 gem_words.cuh step loop", d_ops, d_cnt, d_out, G);
        run<6>("V6 bounds 2 ahead, next ops at step start", d_ops, d_cnt, d_out, G);
        run<7>("V7 V5 + asm-volatile bound move", d_ops, d_cnt, d_out, G);
        run<8>("V8 V5 without the 4-round path", d_ops, d_cnt, d_out, G);
        run<9>("V9 V5 with one-round op prefetch", d_ops, d_cnt, d_out, G);
        run<10>("V10 V8 + V9", d_ops, d_cnt, d_out, G);
        run<11>("V11 V6 one round only", d_ops, d_cnt, d_out, G);
        run<12>("V12 V6 with <= 2 rounds", d_ops, d_cnt, d_out, G);
        for (int i = 0; i < NSTEPS + 2; i++) st[i] = i < NSTEPS ? (uint32_t)(i * fill) | ((uint32_t)fill << 16) : 0u;
        cudaMemcpy(d_cnt, st.data(), st.size() * 4, cudaMemcpyHostToDevice);
        run<13>("V13 packed table, addresses prepared a step ahead", d_ops, d_cnt, d_out, G);
        run<14>("V14 V13 unroll 4 (runtime step count)", d_ops, d_cnt, d_out, G);
        run<15>("V15 V13 unroll 2 (runtime step count)", d_ops, d_cnt, d_out, G);
        run<16>("V16 V13 with operand loads first", d_ops, d_cnt, d_out, G);
        run<17>("V17 packed table, op consumed after barrier", d_ops, d_cnt, d_out, G);
        {
          std::vector<uint32_t> t2((NSTEPS + 2) * 2);
          for (int i = 0; i < NSTEPS + 1; i++) { t2[2 * i] = (uint32_t)(std::min(i, NSTEPS) * fill); t2[2 * i + 1] = i < NSTEPS ? (uint32_t)fill : 0u; }
          cudaMemcpy(d_cnt, t2.data(), t2.size() * 4, cudaMemcpyHostToDevice);
        }
        run<18>("V18 WRD2 loop (uniform 2-level form, 1-level ops)", d_ops, d_cnt, d_out, G);
        run<19>("V19 V18 + idle warps skip op and prefetch", d_ops, d_cnt, d_out, G);
      }
      cudaFree(d_ops);
      cudaFree(d_cnt);
      cudaFree(d_out);
    }
  return 0;
}
