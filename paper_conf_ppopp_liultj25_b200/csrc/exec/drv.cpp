// Driver-API shim for the peer transport (see drv.h).
#include "drv.h"

#include <cuda.h>
#include <cudaTypedefs.h>

#include <mutex>

namespace mario {
namespace drv {
namespace {

template <class F>
F sym(const char* name) {
  void* p = nullptr;
  cudaDriverEntryPointQueryResult q;
  if (cudaGetDriverEntryPointByVersion(name, &p, 12080, cudaEnableDefault, &q) != cudaSuccess ||
      q != cudaDriverEntryPointSuccess)
    return nullptr;
  return reinterpret_cast<F>(p);
}

struct Api {
  PFN_cuStreamWaitValue32_v8000 wait = nullptr;
  PFN_cuStreamWriteValue32_v8000 write = nullptr;
  PFN_cuDeviceGetDevResource_v12040 get_res = nullptr;
  PFN_cuDevSmResourceSplitByCount_v12040 split = nullptr;
  PFN_cuDevResourceGenerateDesc_v12040 gen_desc = nullptr;
  PFN_cuGreenCtxCreate_v12040 gc_create = nullptr;
  PFN_cuGreenCtxDestroy_v12040 gc_destroy = nullptr;
  PFN_cuGreenCtxStreamCreate_v12050 gc_stream = nullptr;
  PFN_cuGetErrorString_v6000 err = nullptr;
};

const Api& api() {
  static Api a;
  static std::once_flag once;
  std::call_once(once, [] {
    a.wait = sym<PFN_cuStreamWaitValue32_v8000>("cuStreamWaitValue32");
    a.write = sym<PFN_cuStreamWriteValue32_v8000>("cuStreamWriteValue32");
    a.get_res = sym<PFN_cuDeviceGetDevResource_v12040>("cuDeviceGetDevResource");
    a.split = sym<PFN_cuDevSmResourceSplitByCount_v12040>("cuDevSmResourceSplitByCount");
    a.gen_desc = sym<PFN_cuDevResourceGenerateDesc_v12040>("cuDevResourceGenerateDesc");
    a.gc_create = sym<PFN_cuGreenCtxCreate_v12040>("cuGreenCtxCreate");
    a.gc_destroy = sym<PFN_cuGreenCtxDestroy_v12040>("cuGreenCtxDestroy");
    a.gc_stream = sym<PFN_cuGreenCtxStreamCreate_v12050>("cuGreenCtxStreamCreate");
    a.err = sym<PFN_cuGetErrorString_v6000>("cuGetErrorString");
  });
  return a;
}

std::string errstr(CUresult r) {
  const char* s = nullptr;
  if (api().err) api().err(r, &s);
  return s ? s : ("CUresult " + std::to_string(static_cast<int>(r)));
}

std::vector<CUgreenCtx> g_ctxs;

}  // namespace

cudaError_t wait_flag(cudaStream_t s, const uint32_t* addr, uint32_t value) {
  if (!api().wait) return cudaErrorNotSupported;
  return api().wait(reinterpret_cast<CUstream>(s), reinterpret_cast<CUdeviceptr>(addr), value,
                    CU_STREAM_WAIT_VALUE_GEQ) == CUDA_SUCCESS
             ? cudaSuccess
             : cudaErrorUnknown;
}

cudaError_t write_flag(cudaStream_t s, uint32_t* addr, uint32_t value) {
  if (!api().write) return cudaErrorNotSupported;
  return api().write(reinterpret_cast<CUstream>(s), reinterpret_cast<CUdeviceptr>(addr), value,
                     CU_STREAM_WRITE_VALUE_DEFAULT) == CUDA_SUCCESS
             ? cudaSuccess
             : cudaErrorUnknown;
}

std::string make_partitions(int device, int n, int sms, int per_part, std::vector<std::vector<cudaStream_t>>& streams,
                            int* sms_actual) {
  const Api& a = api();
  if (!a.get_res || !a.split || !a.gen_desc || !a.gc_create || !a.gc_stream) return "green-context API unavailable";
  CUdevResource all{};
  CUresult r = a.get_res(static_cast<CUdevice>(device), &all, CU_DEV_RESOURCE_TYPE_SM);
  if (r != CUDA_SUCCESS) return "cuDeviceGetDevResource: " + errstr(r);
  std::vector<CUdevResource> parts(n);
  unsigned got = static_cast<unsigned>(n);
  CUdevResource rem{};
  r = a.split(parts.data(), &got, &all, &rem, 0, static_cast<unsigned>(sms));
  if (r != CUDA_SUCCESS) return "cuDevSmResourceSplitByCount: " + errstr(r);
  if (static_cast<int>(got) < n)
    return "only " + std::to_string(got) + " partitions of " + std::to_string(sms) + " SMs fit on the device";
  streams.assign(n, {});
  for (int i = 0; i < n; ++i) {
    CUdevResourceDesc desc;
    r = a.gen_desc(&desc, &parts[i], 1);
    if (r != CUDA_SUCCESS) return "cuDevResourceGenerateDesc: " + errstr(r);
    CUgreenCtx gc;
    r = a.gc_create(&gc, desc, static_cast<CUdevice>(device), CU_GREEN_CTX_DEFAULT_STREAM);
    if (r != CUDA_SUCCESS) return "cuGreenCtxCreate: " + errstr(r);
    g_ctxs.push_back(gc);
    for (int j = 0; j < per_part; ++j) {
      CUstream s;
      r = a.gc_stream(&s, gc, CU_STREAM_NON_BLOCKING, 0);
      if (r != CUDA_SUCCESS) return "cuGreenCtxStreamCreate: " + errstr(r);
      streams[i].push_back(reinterpret_cast<cudaStream_t>(s));
    }
  }
  if (sms_actual) *sms_actual = static_cast<int>(parts[0].sm.smCount);
  return "";
}

void destroy_partitions() {
  // streams created in a green context are released with it
  for (CUgreenCtx c : g_ctxs)
    if (api().gc_destroy) api().gc_destroy(c);
  g_ctxs.clear();
}

}  // namespace drv
}  // namespace mario
