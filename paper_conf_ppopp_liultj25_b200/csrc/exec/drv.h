// Driver-API pieces the peer transport needs, resolved at run time through the runtime's
// driver entry points (no link-time libcuda dependency):
//  - stream memory operations (cuStreamWaitValue32 / cuStreamWriteValue32): a receive waits on a
//    flag the sender's stream writes after its data, entirely on the device (no host round trip);
//  - green contexts (cuGreenCtxCreate over an SM split): an emulated pipeline runs every stage's
//    streams on a disjoint SM partition of one GPU.
#pragma once
#include <cuda_runtime.h>

#include <cstdint>
#include <string>
#include <vector>

namespace mario {
namespace drv {

// 32-bit flags in device memory. wait: the stream stalls until *addr >= value.
// write: *addr = value after all prior work of the stream (with a memory fence).
cudaError_t wait_flag(cudaStream_t s, const uint32_t* addr, uint32_t value);
cudaError_t write_flag(cudaStream_t s, uint32_t* addr, uint32_t value);

// Split the device's SMs into n partitions of `sms` SMs (the driver rounds to its granularity:
// multiples of 8 on sm_90+) and create `per_part` non-blocking streams in each partition's green
// context. On success returns "" and the SM count each partition actually got; otherwise an error
// message. The green contexts live until destroy_partitions().
std::string make_partitions(int device, int n, int sms, int per_part, std::vector<std::vector<cudaStream_t>>& streams,
                            int* sms_actual);
void destroy_partitions();

}  // namespace drv
}  // namespace mario
