// Launch accounting and optional per-kernel-class CUDA-event timing (for bench.py's roofline:
// achieved = algorithmic FLOPs / measured launch duration, on the launching stream).
#pragma once
#include <cuda_runtime.h>

namespace mario {
enum KKind { K_GEMM = 0, K_ATTN_FWD = 1, K_ATTN_BWD = 2, K_OTHER = 3, K_NORM = 4, K_COLSUM = 5, K_CE = 6,
             K_ELEMWISE = 7, K_EMBED = 8, K_NKINDS = 9 };

void note_launch(int n = 1);
bool kstats_on();
long long kstats_generation();   // bumped by every mario_kstats_enable (invalidates captured graphs)
// returns a token to pass to kstats_end (or -1 when disabled)
int kstats_begin(KKind kind, double flops, double bytes, cudaStream_t st);
void kstats_end(int token, cudaStream_t st);

// RAII helper: times one launcher when statistics are on
struct KScope {
  int tok;
  cudaStream_t st;
  KScope(KKind k, cudaStream_t s, double bytes = 0.0) : tok(kstats_begin(k, 0.0, bytes, s)), st(s) {}
  ~KScope() { kstats_end(tok, st); }
};
}  // namespace mario
