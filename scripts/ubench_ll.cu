// Micro-benchmark: per-cycle flop exchange without a grid barrier ("LL":
// every committed word carries its cycle tag in the same 8-byte store; a
// reader polls its input-port words until the tag matches), against the flat
// barrier + port loads of gem_runtime.cu (ubench_ports.cu: ~3.4K clk).
// 135 CTAs x 256 threads, 1024 flop words, each CTA owns ~8 words and reads
// 313 random ones per cycle (C3's mean port count).  Buffers: 3 (tag t in
// buffer t % 3); a writer of cycle t+1 may overwrite the buffer of cycle t-2
// only when every CTA has finished reading cycle t-2's ports: each CTA
// publishes its read progress, a writer checks the minimum before its commit
// (loads issued at the top of its cycle, so the check costs no latency unless
// a reader is two cycles behind).
// Build/run: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/ull scripts/ubench_ll.cu && /tmp/ull
#include <cstdint>
#include <cstdio>
#include <vector>
#include <random>
#include <algorithm>

#define NT 256
#define QW 1024
#define NG 313
#define STRIDE 16

__device__ __forceinline__ unsigned long long ld_rlx(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_rlx(unsigned long long* p, unsigned long long v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

// GUARD: 1 = progress check before the commit (the real protocol)
template <int GUARD>
__global__ void __launch_bounds__(NT, 1) k(unsigned long long* q, const uint16_t* __restrict__ gidx,
                                           unsigned long long* prog, unsigned long long* out, int cycles, int work) {
  __shared__ uint32_t S[2048];
  const uint32_t tid = threadIdx.x, B = blockIdx.x, G = gridDim.x;
  uint32_t idx[2];
  for (int u = 0; u < 2; u++) {
    const uint32_t kk = u * NT + tid;
    idx[u] = kk < NG ? gidx[B * NG + kk] : 0xFFFFu;
  }
  const uint32_t own0 = B * QW / G, own1 = (B + 1) * QW / G;
  unsigned long long tot = 0, t0 = 0;
  uint32_t acc = 0;
  for (int c = 1; c < cycles; c++) {
    if (c == 10) t0 = clock64();
    // guard loads for this cycle's commit (min progress >= c - 1, i.e. every CTA read cycle c-1's
    // ports, so buffer (c+1) % 3 == (c-2) % 3 is free)
    unsigned long long gp = ~0ull;
    if (GUARD)
      for (uint32_t f = tid; f < G; f += NT) gp = ld_rlx(prog + (size_t)f * STRIDE);
    // ports of cycle c: poll until tagged c
    const unsigned long long* Qc = q + (size_t)(c % 3) * QW;
#pragma unroll
    for (int u = 0; u < 2; u++) {
      if (idx[u] == 0xFFFFu) continue;
      unsigned long long v;
      do { v = ld_rlx(Qc + idx[u]); } while ((v >> 32) != (unsigned long long)c);
      S[(u * NT + tid) & 2047] = (uint32_t)v;
    }
    __syncthreads();
    if (tid == 0) st_rlx(prog + (size_t)B * STRIDE, (unsigned long long)c);   // read progress
    // "steps": a short dependent chain standing for the layers
    uint32_t x = S[tid];
    for (int w = 0; w < work; w++) { x = S[(x + tid) & 2047] ^ (x << 1); __syncthreads(); }
    acc += x;
    if (GUARD) {
      for (uint32_t f = tid; f < G; f += NT)
        while (gp < (unsigned long long)(c - 1)) gp = ld_rlx(prog + (size_t)f * STRIDE);
      __syncthreads();
    }
    // commit cycle c+1's owned words, tagged c+1
    unsigned long long* Qn = q + (size_t)((c + 1) % 3) * QW;
    for (uint32_t w = own0 + tid; w < own1; w += NT)
      st_rlx(Qn + w, ((unsigned long long)(c + 1) << 32) | (uint32_t)(S[w & 2047] + c + acc));
    if (c >= 10) tot = clock64() - t0;
  }
  if (tid == 0) out[B] = tot / (cycles - 10);
  if (acc == 0x7777777u) out[G + B] = acc;
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
  unsigned long long *d_q, *d_prog, *d_out;
  cudaMalloc(&d_idx, idx.size() * 2);
  cudaMemcpy(d_idx, idx.data(), idx.size() * 2, cudaMemcpyHostToDevice);
  cudaMalloc(&d_q, 3 * QW * 8);
  cudaMalloc(&d_prog, 1024 * STRIDE * 8);
  cudaMalloc(&d_out, 2 * G * 8);
  for (int work : {0, 20}) {
    for (int guard = 0; guard < 2; guard++) {
      // initial state: cycle 1's words tagged 1 in buffer 1
      std::vector<unsigned long long> q0(3 * QW, 0);
      for (int w = 0; w < QW; w++) q0[1 * QW + w] = (1ull << 32) | (uint32_t)w;
      cudaMemcpy(d_q, q0.data(), q0.size() * 8, cudaMemcpyHostToDevice);
      cudaMemset(d_prog, 0, 1024 * STRIDE * 8);
      void* args[] = {&d_q, &d_idx, &d_prog, &d_out, nullptr, nullptr};
      int cycles = 2010;
      args[4] = &cycles;
      args[5] = &work;
      cudaError_t e = guard ? cudaLaunchCooperativeKernel((const void*)k<1>, G, NT, args, 0, 0)
                            : cudaLaunchCooperativeKernel((const void*)k<0>, G, NT, args, 0, 0);
      cudaError_t e2 = cudaDeviceSynchronize();
      std::vector<unsigned long long> h(G);
      cudaMemcpy(h.data(), d_out, G * 8, cudaMemcpyDeviceToHost);
      double m = 0, mx = 0;
      for (auto x : h) { m += x; mx = std::max(mx, (double)x); }
      printf("LL exchange, guard %d, work %2d: %6.0f clk/cycle (max %6.0f)  (%s / %s)\n", guard, work, m / G, mx,
             cudaGetErrorString(e), cudaGetErrorString(e2));
    }
  }
  return 0;
}
