#include "kstats.h"

#include <atomic>
#include <mutex>
#include <vector>

#include "../../../include/mario_kernels.h"

namespace mario {
namespace {
std::atomic<long long> g_launches{0};
bool g_on = false;
unsigned g_mask = 0;   // bit k: time kind k
long long g_gen = 0;
struct Rec { int kind; double flops, bytes; cudaEvent_t a, b; bool captured; };
std::vector<Rec> g_recs;
std::mutex g_mu;
}  // namespace

void note_launch(int n) { g_launches.fetch_add(n, std::memory_order_relaxed); }
bool kstats_on() { return g_on; }
long long kstats_generation() { return g_gen; }

int kstats_begin(KKind kind, double flops, double bytes, cudaStream_t st) {
  if (!g_on || !((g_mask >> kind) & 1u)) return -1;
  std::lock_guard<std::mutex> lk(g_mu);
  cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
  cudaStreamIsCapturing(st, &cs);
  Rec r{kind, flops, bytes, nullptr, nullptr, cs == cudaStreamCaptureStatusActive};
  cudaEventCreate(&r.a);
  cudaEventCreate(&r.b);
  // inside a capture only an External record becomes a graph node that records on every replay
  cudaEventRecordWithFlags(r.a, st, r.captured ? cudaEventRecordExternal : cudaEventRecordDefault);
  g_recs.push_back(r);
  return static_cast<int>(g_recs.size()) - 1;
}

void kstats_end(int token, cudaStream_t st) {
  if (token < 0) return;
  std::lock_guard<std::mutex> lk(g_mu);
  cudaEventRecordWithFlags(g_recs[token].b, st, g_recs[token].captured ? cudaEventRecordExternal : cudaEventRecordDefault);
}
}  // namespace mario

using namespace mario;

extern "C" long long mario_kernel_launches(void) { return g_launches.load(); }

extern "C" int mario_kstats_enable(int mask) {
  std::lock_guard<std::mutex> lk(g_mu);
  for (auto& r : g_recs) { cudaEventDestroy(r.a); cudaEventDestroy(r.b); }
  g_recs.clear();
  g_mask = static_cast<unsigned>(mask);
  ++g_gen;
  g_on = mask != 0;
  return 0;
}

extern "C" int mario_kstats_read(int kind, double* total_ms, double* flops, double* bytes, long long* launches) {
  std::lock_guard<std::mutex> lk(g_mu);
  double ms = 0, fl = 0, by = 0;
  long long n = 0;
  // records captured into a CUDA graph are re-recorded by every replay: when present, they alone
  // are read (the latest replay); otherwise the eager records
  bool any_captured = false;
  for (auto& r : g_recs) any_captured = any_captured || (r.kind == kind && r.captured);
  for (auto& r : g_recs) {
    if (r.kind != kind || r.captured != any_captured) continue;
    float t = 0.f;
    if (cudaEventSynchronize(r.b) != cudaSuccess || cudaEventElapsedTime(&t, r.a, r.b) != cudaSuccess) return -1;
    ms += t; fl += r.flops; by += r.bytes; ++n;
  }
  if (total_ms) *total_ms = ms;
  if (flops) *flops = fl;
  if (bytes) *bytes = by;
  if (launches) *launches = n;
  return 0;
}
