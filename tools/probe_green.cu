// Probe: can one B200 host S concurrently running "pipeline stages" on disjoint SM partitions?
// Green contexts (driver API) + runtime-API launches into their streams, stream memory ops
// (cuStreamWaitValue32 / cuStreamWriteValue32) for cross-stream flags, cluster launches, and
// CUDA-graph capture across the partitioned streams.
//   nvcc -gencode arch=compute_100a,code=sm_100a -o /tmp/probe_green tools/probe_green.cu
#include <cuda.h>
#include <cuda_runtime.h>
#include <cudaTypedefs.h>
#include <cstdio>
#include <set>
#include <vector>
#define printf(...) (fprintf(stderr, __VA_ARGS__), fflush(stderr))

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("FAIL %s: %s\n", #x, cudaGetErrorString(e)); return 1; } } while (0)
#define DK(x) do { CUresult e = (x); if (e != CUDA_SUCCESS) { const char* s; cuGetErrorString_(e, &s); printf("FAIL %s: %s\n", #x, s); return 1; } } while (0)

static PFN_cuGetErrorString_v6000 cuGetErrorString_;

template <class F> F sym(const char* name) {
  void* p = nullptr;
  cudaDriverEntryPointQueryResult q;
  if (cudaGetDriverEntryPointByVersion(name, &p, 12080, cudaEnableDefault, &q) != cudaSuccess || !p) {
    printf("no driver symbol %s\n", name);
    return nullptr;
  }
  return reinterpret_cast<F>(p);
}

__global__ void smid_k(int* out, int spin) {
  unsigned s;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(s));
  if (threadIdx.x == 0) out[blockIdx.x] = s;
  long long t0 = clock64();
  while (clock64() - t0 < spin) {}
}
__global__ void __cluster_dims__(2, 1, 1) cluster_k(int* out) {
  unsigned s, r;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(s));
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  if (threadIdx.x == 0) out[blockIdx.x] = s * 2 + r;
}
__global__ void stamp_k(unsigned long long* out) {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  *out = t;
}

int main() {
  CK(cudaSetDevice(0));
  CK(cudaFree(0));
  cuGetErrorString_ = sym<PFN_cuGetErrorString_v6000>("cuGetErrorString");
  auto getRes = sym<PFN_cuDeviceGetDevResource_v12040>("cuDeviceGetDevResource");
  auto split = sym<PFN_cuDevSmResourceSplitByCount_v12040>("cuDevSmResourceSplitByCount");
  auto genDesc = sym<PFN_cuDevResourceGenerateDesc_v12040>("cuDevResourceGenerateDesc");
  auto gcCreate = sym<PFN_cuGreenCtxCreate_v12040>("cuGreenCtxCreate");
  auto gcStream = sym<PFN_cuGreenCtxStreamCreate_v12050>("cuGreenCtxStreamCreate");
  auto waitV = sym<PFN_cuStreamWaitValue32_v8000>("cuStreamWaitValue32");
  auto writeV = sym<PFN_cuStreamWriteValue32_v8000>("cuStreamWriteValue32");
  if (!getRes || !split || !genDesc || !gcCreate || !gcStream || !waitV || !writeV) return 1;
  CUdevice dev = 0;
  CUdevResource all;
  DK(getRes(dev, &all, CU_DEV_RESOURCE_TYPE_SM));
  printf("device SMs: %u\n", all.sm.smCount);
  printf("step: split\n");
  const int G = 8;
  for (unsigned minc : {16u, 18u}) {
    std::vector<CUdevResource> parts(G);
    unsigned n = G;
    CUdevResource rem;
    CUresult r = split(parts.data(), &n, &all, &rem, 0, minc);
    printf("split min %u -> %s groups %u, sm each %u, remaining %u\n", minc, r == CUDA_SUCCESS ? "ok" : "ERR", n,
           n ? parts[0].sm.smCount : 0, rem.sm.smCount);
  }
  std::vector<CUdevResource> parts(G);
  unsigned n = G;
  CUdevResource rem;
  DK(split(parts.data(), &n, &all, &rem, 0, 16));
  std::vector<CUstream> st(n);
  for (unsigned i = 0; i < n; ++i) {
    CUdevResourceDesc d;
    DK(genDesc(&d, &parts[i], 1));
    CUgreenCtx gc;
    DK(gcCreate(&gc, d, dev, CU_GREEN_CTX_DEFAULT_STREAM));
    DK(gcStream(&st[i], gc, CU_STREAM_NON_BLOCKING, 0));
  }
  // 1) runtime launches into green streams stay inside the partition, partitions disjoint
  const int B = 2048;
  int* d_sm;
  CK(cudaMalloc(&d_sm, sizeof(int) * B * n));
  for (unsigned i = 0; i < n; ++i) smid_k<<<B, 128, 0, (cudaStream_t)st[i]>>>(d_sm + i * B, 20000);
  CK(cudaDeviceSynchronize());
  std::vector<int> h(B * n);
  CK(cudaMemcpy(h.data(), d_sm, sizeof(int) * B * n, cudaMemcpyDeviceToHost));
  std::set<int> seen;
  bool disjoint = true;
  for (unsigned i = 0; i < n; ++i) {
    std::set<int> s(h.begin() + i * B, h.begin() + (i + 1) * B);
    for (int x : s) if (seen.count(x)) disjoint = false;
    seen.insert(s.begin(), s.end());
    printf("partition %u: %zu distinct SMs (min %d max %d)\n", i, s.size(), *s.begin(), *s.rbegin());
  }
  printf("RESULT partitions_disjoint=%d total_sms_used=%zu\n", (int)disjoint, seen.size());
  // 2) cluster launch in a green stream
  cluster_k<<<64, 64, 0, (cudaStream_t)st[1]>>>(d_sm);
  cudaError_t ce = cudaDeviceSynchronize();
  printf("RESULT cluster_launch=%s\n", cudaGetErrorString(ce));
  // 3) cross-stream flag: st[0] waits flag >= 1 then stamps; st[1] spins ~20 ms then writes the flag
  unsigned* flag;
  unsigned long long* stamps;
  CK(cudaMalloc(&flag, 4));
  CK(cudaMalloc(&stamps, 16));
  CK(cudaMemset(flag, 0, 4));
  CK(cudaDeviceSynchronize());
  // the write is ENQUEUED before the wait (the executor's rule), but executes ~20 ms later
  smid_k<<<16, 32, 0, (cudaStream_t)st[1]>>>(d_sm, 40000000);
  stamp_k<<<1, 1, 0, (cudaStream_t)st[1]>>>(stamps + 1);
  DK(writeV(st[1], (CUdeviceptr)flag, 1, 0));
  DK(waitV(st[0], (CUdeviceptr)flag, 1, CU_STREAM_WAIT_VALUE_GEQ));
  stamp_k<<<1, 1, 0, (cudaStream_t)st[0]>>>(stamps);
  CK(cudaDeviceSynchronize());
  unsigned long long hs[2];
  CK(cudaMemcpy(hs, stamps, 16, cudaMemcpyDeviceToHost));
  printf("RESULT wait_value_ordered=%d (waiter - writer-side stamp = %lld ns)\n", (int)(hs[0] >= hs[1]),
         (long long)(hs[0] - hs[1]));
  // 4) graph capture across green streams (fork/join with events) + memops in the graph
  cudaStream_t origin;
  CK(cudaStreamCreateWithFlags(&origin, cudaStreamNonBlocking));
  cudaEvent_t ef, ej[8];
  CK(cudaEventCreateWithFlags(&ef, cudaEventDisableTiming));
  for (auto& ev : ej) CK(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
  CK(cudaMemset(flag, 0, 4));
  CK(cudaMemset(d_sm, 0xff, sizeof(int) * B * n));
  CK(cudaDeviceSynchronize());
  CK(cudaStreamBeginCapture(origin, cudaStreamCaptureModeThreadLocal));
  CK(cudaEventRecord(ef, origin));
  for (unsigned i = 0; i < n; ++i) CK(cudaStreamWaitEvent((cudaStream_t)st[i], ef, 0));
  smid_k<<<B, 128, 0, (cudaStream_t)st[1]>>>(d_sm + 1 * B, 20000);
  DK(writeV(st[1], (CUdeviceptr)flag, 1, 0));
  DK(waitV(st[0], (CUdeviceptr)flag, 1, CU_STREAM_WAIT_VALUE_GEQ));
  for (unsigned i = 0; i < n; ++i) {
    if (i != 1) smid_k<<<B, 128, 0, (cudaStream_t)st[i]>>>(d_sm + i * B, 20000);
    CK(cudaEventRecord(ej[i], (cudaStream_t)st[i]));
    CK(cudaStreamWaitEvent(origin, ej[i], 0));
  }
  cudaGraph_t gr;
  cudaError_t e1 = cudaStreamEndCapture(origin, &gr);
  printf("RESULT graph_capture=%s\n", cudaGetErrorString(e1));
  if (e1 == cudaSuccess) {
    cudaGraphExec_t ex;
    CK(cudaGraphInstantiate(&ex, gr, 0));
    CK(cudaGraphLaunch(ex, origin));
    CK(cudaStreamSynchronize(origin));
    CK(cudaMemcpy(h.data(), d_sm, sizeof(int) * B * n, cudaMemcpyDeviceToHost));
    std::set<int> seen2;
    bool dis2 = true;
    for (unsigned i = 0; i < n; ++i) {
      std::set<int> s(h.begin() + i * B, h.begin() + (i + 1) * B);
      for (int x : s) if (seen2.count(x)) dis2 = false;
      seen2.insert(s.begin(), s.end());
      printf("graph partition %u: %zu SMs\n", i, s.size());
    }
    printf("RESULT graph_partitions_disjoint=%d\n", (int)dis2);
  }
  printf("PROBE DONE\n");
  return 0;
}
