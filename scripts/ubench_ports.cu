// Micro-benchmark: the per-cycle exchange of the single-stream path without
// the layers -- every CTA commits its owned flop words, meets the others at
// the flat flag barrier (as in gem_runtime.cu grid_sync), then loads its input
// ports (~313 of 1024 words, C3's mean gread) from L2 into shared memory.
// Answers: how much of C3's ~2.5K clk "ports" phase is the L2 exchange itself,
// and does spreading the Q words over more L2 lines/slices (stride SP words)
// or replicating them (R copies, reader b reads copy b % R) change it?
// Build/run: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/up scripts/ubench_ports.cu && /tmp/up
#include <cstdint>
#include <cstdio>
#include <vector>
#include <random>
#include <algorithm>

#define NT 256
#define QW 1024
#define NG 313
#define STRIDE 16   // u64 words between barrier flags

__device__ __forceinline__ unsigned long long ld_acq(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_rel(unsigned long long* p, unsigned long long v) {
  asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ unsigned long long ld_rlx(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void red_rel(unsigned long long* p, unsigned long long v) {
  asm volatile("red.release.gpu.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// BM (barrier mode): 0 flat flags, st.release + ld.acquire polls (product);
// 1 flat flags, relaxed polls + one fence.acq_rel.gpu per polling thread;
// 2 flat flags polled by warp 0..4 only, relaxed + fence;
// 3 single counter: red.release.add by thread 0, thread 0 polls ld.acquire;
// 4 single counter, relaxed poll + fence;
// 5 flat flags, fence.acq_rel + st.relaxed arrive, relaxed polls + fence
template <int SP, int R, int BM>
__global__ void __launch_bounds__(NT, 1) k(uint32_t* q, const uint16_t* __restrict__ gidx, unsigned long long* bar,
                                           unsigned long long* out, int cycles) {
  __shared__ uint32_t S[2048];
  const uint32_t tid = threadIdx.x, B = blockIdx.x, G = gridDim.x;
  // this CTA's port list (in registers, like the resident program)
  uint32_t idx[2];
  for (int u = 0; u < 2; u++) {
    const uint32_t kk = u * NT + tid;
    idx[u] = kk < NG ? gidx[B * NG + kk] : 0xFFFFu;
  }
  const uint32_t own0 = B * QW / G, own1 = (B + 1) * QW / G;
  unsigned long long ep = 0, tl = 0, tb = 0, tc = 0;
  uint32_t acc = 0;
  for (int c = 0; c < cycles; c++) {
    const uint32_t cur = c & 1, nxt = cur ^ 1;
    const uint32_t* Qc = q + (size_t)cur * QW * SP * R + (B % R) * QW * SP;
    unsigned long long t0 = clock64();
    uint32_t v[2];
#pragma unroll
    for (int u = 0; u < 2; u++) v[u] = idx[u] != 0xFFFFu ? __ldcg(Qc + idx[u] * SP) : 0u;
#pragma unroll
    for (int u = 0; u < 2; u++) if (idx[u] != 0xFFFFu) S[(u * NT + tid) & 2047] = v[u];
    __syncthreads();
    unsigned long long t1 = clock64();
    // "layers": none; commit: owned words of the next cycle (all R copies)
    for (uint32_t w = own0 + tid; w < own1; w += NT) {
      const uint32_t val = S[w & 2047] + c;
      for (int r = 0; r < R; r++) __stcg(q + (size_t)nxt * QW * SP * R + r * QW * SP + w * SP, val);
    }
    unsigned long long t2 = clock64();
    __syncthreads();
    ep++;
    if (BM == 0) {
      if (tid == 0) st_rel(bar + (size_t)B * STRIDE, ep);
      for (uint32_t f = tid; f < G; f += NT)
        while (ld_acq(bar + (size_t)f * STRIDE) < ep) {}
    } else if (BM == 1 || BM == 2 || BM == 5) {
      if (tid == 0) {
        if (BM == 5) {
          asm volatile("fence.acq_rel.gpu;" ::: "memory");
          asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(bar + (size_t)B * STRIDE), "l"(ep) : "memory");
        } else {
          st_rel(bar + (size_t)B * STRIDE, ep);
        }
      }
      const uint32_t np = BM == 2 ? 160u : NT;
      if (tid < np) {
        for (uint32_t f = tid; f < G; f += np)
          while (ld_rlx(bar + (size_t)f * STRIDE) < ep) {}
        asm volatile("fence.acq_rel.gpu;" ::: "memory");
      }
    } else {
      if (tid == 0) {
        red_rel(bar, 1ull);
        if (BM == 3) { while (ld_acq(bar) < ep * G) {} }
        else { while (ld_rlx(bar) < ep * G) {} asm volatile("fence.acq_rel.gpu;" ::: "memory"); }
      }
    }
    __syncthreads();
    unsigned long long t3 = clock64();
    if (c >= 10) { tl += t1 - t0; tc += t2 - t1; tb += t3 - t2; }
    acc += S[tid];
  }
  if (tid == 0) {
    out[B * 4 + 0] = tl / (cycles - 10);
    out[B * 4 + 1] = tc / (cycles - 10);
    out[B * 4 + 2] = tb / (cycles - 10);
  }
  if (acc == 0x9999999u) out[B * 4 + 3] = acc;
}

template <int SP, int R, int BM = 0>
void run(const char* name, int G, const uint16_t* d_idx, uint32_t* d_q, unsigned long long* d_bar,
         unsigned long long* d_out) {
  cudaMemset(d_bar, 0, 1024 * STRIDE * 8);
  k<SP, R, BM><<<G, NT>>>(d_q, d_idx, d_bar, d_out, 50);
  cudaMemset(d_bar, 0, 1024 * STRIDE * 8);
  k<SP, R, BM><<<G, NT>>>(d_q, d_idx, d_bar, d_out, 2010);
  cudaError_t e = cudaDeviceSynchronize();
  std::vector<unsigned long long> h(G * 4);
  cudaMemcpy(h.data(), d_out, G * 32, cudaMemcpyDeviceToHost);
  double l = 0, c = 0, b = 0, lmax = 0;
  for (int i = 0; i < G; i++) { l += h[i * 4]; c += h[i * 4 + 1]; b += h[i * 4 + 2]; lmax = std::max(lmax, (double)h[i * 4]); }
  printf("%-28s ports %6.0f (max %6.0f)  commit %5.0f  barrier %6.0f  total %6.0f clk  (%s)\n", name, l / G, lmax,
         c / G, b / G, (l + c + b) / G, cudaGetErrorString(e));
}

int main() {
  const int G = 135;
  std::mt19937 rng(7);
  std::vector<uint16_t> idx(G * NG);
  for (int b = 0; b < G; b++) {
    std::vector<uint16_t> all(QW);
    for (int i = 0; i < QW; i++) all[i] = i;
    std::shuffle(all.begin(), all.end(), rng);
    std::sort(all.begin(), all.begin() + NG);
    for (int i = 0; i < NG; i++) idx[b * NG + i] = all[i];
  }
  uint16_t* d_idx;
  uint32_t* d_q;
  unsigned long long *d_bar, *d_out;
  cudaMalloc(&d_idx, idx.size() * 2);
  cudaMemcpy(d_idx, idx.data(), idx.size() * 2, cudaMemcpyHostToDevice);
  cudaMalloc(&d_q, (size_t)2 * QW * 32 * 8 * 4);
  cudaMemset(d_q, 0, (size_t)2 * QW * 32 * 8 * 4);
  cudaMalloc(&d_bar, 1024 * STRIDE * 8);
  cudaMalloc(&d_out, G * 32);
  for (int rep = 0; rep < 2; rep++) {
    run<1, 1>("packed", G, d_idx, d_q, d_bar, d_out);
    run<1, 4>("packed, 4 replicas", G, d_idx, d_q, d_bar, d_out);
    run<1, 1, 1>("bar 1 relaxed poll+fence", G, d_idx, d_q, d_bar, d_out);
    run<1, 1, 2>("bar 2 160 pollers", G, d_idx, d_q, d_bar, d_out);
    run<1, 1, 3>("bar 3 counter acquire", G, d_idx, d_q, d_bar, d_out);
    run<1, 1, 4>("bar 4 counter relaxed", G, d_idx, d_q, d_bar, d_out);
    run<1, 1, 5>("bar 5 fence+relaxed st", G, d_idx, d_q, d_bar, d_out);
  }
  return 0;
}
