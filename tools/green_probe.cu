// Probe: green-context SM partitions driven from the runtime API (sm_100a).  Splits the GPU
// into groups of N SMs, launches a kernel with <<<>>> into a stream of each green context
// (the primary context current) and reports which SMs its blocks ran on.
//   nvcc -gencode arch=compute_100a,code=sm_100a -o green_probe green_probe.cu && ./green_probe 16
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdlib>
#include <set>
#include <vector>

__global__ void where(int *smids, long long spin) {
  int s;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(s));
  const long long t0 = clock64();
  while (clock64() - t0 < spin) {}
  if (threadIdx.x == 0) smids[blockIdx.x] = s;
}

template <class F> F drv(const char *name) {
  void *p = nullptr;
  cudaDriverEntryPointQueryResult q;
  if (cudaGetDriverEntryPoint(name, &p, cudaEnableDefault, &q) != cudaSuccess || q != cudaDriverEntryPointSuccess) {
    printf("no entry point %s\n", name);
    exit(1);
  }
  return (F)p;
}
#define CKD(x) do { CUresult r = (x); if (r != CUDA_SUCCESS) { printf("%s -> %d\n", #x, (int)r); exit(1); } } while (0)

int main(int argc, char **argv) {
  const unsigned want = argc > 1 ? atoi(argv[1]) : 16;
  cudaSetDevice(0);
  cudaFree(0);
  auto pGetRes = drv<CUresult (*)(CUdevice, CUdevResource *, CUdevResourceType)>("cuDeviceGetDevResource");
  auto pSplit = drv<CUresult (*)(CUdevResource *, unsigned *, const CUdevResource *, CUdevResource *, unsigned, unsigned)>("cuDevSmResourceSplitByCount");
  auto pDesc = drv<CUresult (*)(CUdevResourceDesc *, CUdevResource *, unsigned)>("cuDevResourceGenerateDesc");
  auto pCreate = drv<CUresult (*)(CUgreenCtx *, CUdevResourceDesc, CUdevice, unsigned)>("cuGreenCtxCreate");
  auto pStream = drv<CUresult (*)(CUstream *, CUgreenCtx, unsigned, int)>("cuGreenCtxStreamCreate");
  CUdevResource all;
  CKD(pGetRes(0, &all, CU_DEV_RESOURCE_TYPE_SM));
  printf("device SMs %u\n", all.sm.smCount);
  unsigned n = 0;
  CKD(pSplit(nullptr, &n, &all, nullptr, 0, want));
  std::vector<CUdevResource> g(n);
  CUdevResource rem;
  CKD(pSplit(g.data(), &n, &all, &rem, 0, want));
  printf("groups %u of %u SMs, remainder %u\n", n, n ? g[0].sm.smCount : 0, rem.sm.smCount);
  int *d; cudaMalloc(&d, 4096 * sizeof(int));
  std::vector<int> h(4096);
  for (unsigned i = 0; i < n && i < 8; i++) {
    CUdevResourceDesc desc;
    CKD(pDesc(&desc, &g[i], 1));
    CUgreenCtx gc;
    CKD(pCreate(&gc, desc, 0, CU_GREEN_CTX_DEFAULT_STREAM));
    CUstream st;
    CKD(pStream(&st, gc, CU_STREAM_NON_BLOCKING, 0));
    cudaMemset(d, 0xff, 4096 * sizeof(int));
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    cudaEventRecord(e0, (cudaStream_t)st);
    where<<<1024, 128, 0, (cudaStream_t)st>>>(d, 200000);
    cudaEventRecord(e1, (cudaStream_t)st);
    cudaError_t err = cudaStreamSynchronize((cudaStream_t)st);
    float ms = 0; cudaEventElapsedTime(&ms, e0, e1);
    cudaMemcpy(h.data(), d, 1024 * sizeof(int), cudaMemcpyDeviceToHost);
    std::set<int> sms(h.begin(), h.begin() + 1024);
    printf("group %u: err=%s  %.3f ms  distinct SMs %zu  [", i, cudaGetErrorString(err), ms, sms.size());
    int c = 0;
    for (int s : sms) { if (c++ < 20) printf("%d ", s); }
    printf("]\n");
  }
  // reference: the same kernel on a plain stream
  cudaStream_t ps; cudaStreamCreateWithFlags(&ps, cudaStreamNonBlocking);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  cudaEventRecord(e0, ps);
  where<<<1024, 128, 0, ps>>>(d, 200000);
  cudaEventRecord(e1, ps);
  cudaStreamSynchronize(ps);
  float ms = 0; cudaEventElapsedTime(&ms, e0, e1);
  cudaMemcpy(h.data(), d, 1024 * sizeof(int), cudaMemcpyDeviceToHost);
  std::set<int> sms(h.begin(), h.begin() + 1024);
  printf("plain stream: %.3f ms  distinct SMs %zu\n", ms, sms.size());
  return 0;
}
