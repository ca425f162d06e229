// Microbenchmark: per-SM lane-op throughput of the DPX / packed-int16 / int32
// instructions the Gotoh recurrence uses on sm_100a. Prints lane-ops per SM-clock.
// Used to derive the ALU roofline peak in DESIGN.md (R in GCUPS_peak = N_SM f R / I_cell).
#include <cstdio>
#include <cuda_fp16.h>
#include <cstdint>
#include <vector>
#include <algorithm>
#include <map>
#define CHAINS 8
#define ITERS 4096

template <int OP>
__device__ __forceinline__ uint32_t op(uint32_t a, uint32_t b, uint32_t c) {
  if (OP == 0) return __viaddmax_s16x2(a, b, c);
  if (OP == 1) return __vimax3_s16x2_relu(a, b, c);
  if (OP == 2) return __vadd2(a, b);
  if (OP == 3) return __vmaxs2(a, b);
  if (OP == 4) return (uint32_t)__viaddmax_s32((int)a, (int)b, (int)c);
  if (OP == 5) return (uint32_t)__vimax3_s32_relu((int)a, (int)b, (int)c);
  if (OP == 6) return a + b;                 // IADD3
  if (OP == 7) return a * b + c;             // IMAD
  if (OP == 8) return (uint32_t)max((int)a, (int)b);  // VIMNMX
  if (OP == 9) return __viaddmax_s16x2_relu(a, b, c);
  if (OP == 10) return __vimax_s16x2_relu(a, b);
  if (OP == 11) { __half2 x = *reinterpret_cast<__half2*>(&a), y = *reinterpret_cast<__half2*>(&b);
                  __half2 r = __hmax2(x, y); return *reinterpret_cast<uint32_t*>(&r); }
  if (OP == 12) return __viaddmax_s16x2(a, b, c) ^ 0;   // placeholder, mixed below
  if (OP == 13) return (uint32_t)__float_as_uint(fmaxf(__uint_as_float(a), __uint_as_float(b)));
  return a;
}

template <int OP>
__global__ void bench(uint32_t *out, unsigned long long *t, uint32_t seed) {
  uint32_t v[CHAINS];
#pragma unroll
  for (int c = 0; c < CHAINS; c++) v[c] = seed * (threadIdx.x + c + 1);
  uint32_t b = seed ^ 0x00030003u, cc = seed ^ 0x00050005u;
  __syncthreads();
  unsigned long long t0 = clock64();
#pragma unroll 4
  for (int i = 0; i < ITERS; i++) {
#pragma unroll
    for (int c = 0; c < CHAINS; c++) v[c] = op<OP>(v[c], b, cc);
    b += 0x00010001u;  // keep operands live (1 extra op per CHAINS ops)
  }
  __syncthreads();
  unsigned long long t1 = clock64();
  uint32_t r = 0;
#pragma unroll
  for (int c = 0; c < CHAINS; c++) r ^= v[c];
  out[blockIdx.x * blockDim.x + threadIdx.x] = r;
  if (threadIdx.x == 0) {
    unsigned smid; asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
    t[3 * blockIdx.x] = smid; t[3 * blockIdx.x + 1] = t0; t[3 * blockIdx.x + 2] = t1;
  }
}

__global__ void mixk(uint32_t *out, unsigned long long *t, uint32_t seed, int mode) {
  uint32_t v[CHAINS], w[CHAINS];
#pragma unroll
  for (int c = 0; c < CHAINS; c++) { v[c] = seed * (threadIdx.x + c + 1); w[c] = 0x3c003c00u + c; }
  uint32_t b = seed ^ 0x00030003u, cc = seed ^ 0x00050005u;
  __syncthreads();
  unsigned long long t0 = clock64();
#pragma unroll 4
  for (int i = 0; i < ITERS; i++) {
#pragma unroll
    for (int c = 0; c < CHAINS; c++) {
      v[c] = __viaddmax_s16x2(v[c], b, cc);
      if (mode == 1) { __half2 x = *reinterpret_cast<__half2*>(&w[c]), y = *reinterpret_cast<__half2*>(&v[c]);
                       __half2 r = __hmax2(x, y); w[c] = *reinterpret_cast<uint32_t*>(&r); }
      if (mode == 2) w[c] = __vmaxs2(w[c], v[c]);
      if (mode == 3) w[c] = w[c] + v[c];
    }
    b += 0x00010001u;
  }
  __syncthreads();
  unsigned long long t1 = clock64();
  uint32_t r = 0;
#pragma unroll
  for (int c = 0; c < CHAINS; c++) r ^= v[c] ^ w[c];
  out[blockIdx.x * blockDim.x + threadIdx.x] = r;
  if (threadIdx.x == 0) { t[2 * blockIdx.x] = t0; t[2 * blockIdx.x + 1] = t1; }
}
void runmix(const char *name, int nsm, int mode) {
  int threads = 256, blocks = nsm * 8;
  uint32_t *out; unsigned long long *t;
  cudaMalloc(&out, 4 * blocks * threads); cudaMalloc(&t, 16 * blocks);
  mixk<<<blocks, threads>>>(out, t, 7, mode);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  cudaEventRecord(e0);
  mixk<<<blocks, threads>>>(out, t, 7, mode);
  cudaEventRecord(e1); cudaEventSynchronize(e1);
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  double dpx = (double)blocks * threads * ITERS * CHAINS;
  printf("%-26s DPX lane-ops/s = %.1f G  (ms %.3f)\n", name, dpx / (ms * 1e6), ms);
  cudaFree(out); cudaFree(t);
}

template <int OP>
void run(const char *name, int nsm) {
  int threads = 256, blocks_per_sm = 8, blocks = nsm * blocks_per_sm;
  uint32_t *out; unsigned long long *t;
  cudaMalloc(&out, sizeof(uint32_t) * blocks * threads);
  cudaMalloc(&t, sizeof(unsigned long long) * 3 * blocks);
  bench<OP><<<blocks, threads>>>(out, t, 7);
  bench<OP><<<blocks, threads>>>(out, t, 7);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  cudaEventRecord(e0);
  bench<OP><<<blocks, threads>>>(out, t, 7);
  cudaEventRecord(e1); cudaEventSynchronize(e1);
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  std::vector<unsigned long long> h(3 * blocks);
  cudaMemcpy(h.data(), t, h.size() * 8, cudaMemcpyDeviceToHost);
  std::map<int, std::pair<unsigned long long, unsigned long long>> sm;
  std::map<int, int> cnt;
  for (int b = 0; b < blocks; b++) {
    int s = (int)h[3 * b];
    auto it = sm.find(s);
    if (it == sm.end()) sm[s] = {h[3 * b + 1], h[3 * b + 2]};
    else { it->second.first = std::min(it->second.first, h[3*b+1]); it->second.second = std::max(it->second.second, h[3*b+2]); }
    cnt[s]++;
  }
  double sum_rate = 0; int n = 0;
  for (auto &kv : sm) {
    double ops = (double)cnt[kv.first] * threads * ITERS * CHAINS;
    sum_rate += ops / (double)(kv.second.second - kv.second.first); n++;
  }
  double total_ops = (double)blocks * threads * ITERS * CHAINS;
  printf("%-22s lane-ops/clk/SM = %7.2f   (SMs seen %d)  chip Gops/s = %9.1f  ms=%.3f\n", name,
         sum_rate / n, n, total_ops / (ms * 1e6), ms);
  cudaFree(out); cudaFree(t);
}

int main() {
  int dev = 0; cudaDeviceProp p; cudaGetDeviceProperties(&p, dev);
  int clk = 0; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, dev);
  printf("%s  SMs=%d  clockRate(kHz)=%d\n", p.name, p.multiProcessorCount, clk);
  int nsm = p.multiProcessorCount;
  run<0>("viaddmax_s16x2", nsm);
  run<1>("vimax3_s16x2_relu", nsm);
  run<2>("vadd2", nsm);
  run<3>("vmaxs2", nsm);
  run<4>("viaddmax_s32", nsm);
  run<5>("vimax3_s32_relu", nsm);
  run<6>("iadd", nsm);
  run<7>("imad", nsm);
  run<8>("imax_s32", nsm);
  run<9>("viaddmax_s16x2_relu", nsm);
  run<10>("vimax_s16x2_relu", nsm);
  run<11>("hmax2", nsm);
  run<13>("fmaxf", nsm);
  runmix("mix dpx only", nsm, 0);
  runmix("mix dpx + hmax2", nsm, 1);
  runmix("mix dpx + vmaxs2", nsm, 2);
  runmix("mix dpx + iadd", nsm, 3);
  return 0;
}
