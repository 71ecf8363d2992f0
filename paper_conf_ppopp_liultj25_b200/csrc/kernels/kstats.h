// Launch accounting and optional per-kernel-class CUDA-event timing (for bench.py's roofline:
// achieved = algorithmic FLOPs / measured launch duration, on the launching stream).
#pragma once
#include <cuda_runtime.h>

namespace mario {
enum KKind { K_GEMM = 0, K_ATTN_FWD = 1, K_ATTN_BWD = 2, K_OTHER = 3, K_NKINDS = 4 };
void note_launch(int n = 1);
bool kstats_on();
// returns a token to pass to kstats_end (or -1 when disabled)
int kstats_begin(KKind kind, double flops, double bytes, cudaStream_t st);
void kstats_end(int token, cudaStream_t st);
}  // namespace mario
