// comm.h - K5: batch-sharded data parallelism.
// A library-owned NCCL communicator, resolved with dlopen so the library loads (and its CPU
// tests run) without NCCL; over NVLink 5 / NVSwitch on the B200 box.  Two collectives per step:
// allreduce(s_t, int64) before SST so every rank computes the same keep mask, and
// allreduce(dW, fp32) before Adam.
#pragma once
#include <cstddef>
#include <string>
#include <cuda_runtime.h>

namespace sk {

struct Comm {
    void *comm = nullptr;  // ncclComm_t
    int rank = 0, world = 1;
    static bool unique_id(unsigned char id[128], std::string *err);
    bool init(const unsigned char id[128], int rank, int world, std::string *err);
    bool allreduce_i64(long long *buf, size_t n, cudaStream_t s, std::string *err);
    bool allreduce_f32(float *buf, size_t n, cudaStream_t s, std::string *err);
    bool allreduce_f64(double *buf, size_t n, cudaStream_t s, std::string *err);
    void destroy();
};

}  // namespace sk
