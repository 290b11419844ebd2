// dev_util.cuh — RAII helpers for the flow kernels (reduce_gpu.cu, classes_gpu.cu): a device block
// taken from the context's DevPool (no cudaMalloc/cudaFree per call when cached) and a timing
// event pair (device time of the kernels, recorded on the launch stream).
#pragma once
#include <cuda_runtime.h>

#include "cec_internal.hpp"

namespace cec {
struct DevBlock {
    DevPool *pool;
    cudaStream_t st;
    void *p = nullptr;
    size_t cap = 0;
    const char *alloc(size_t bytes) {
        if (pool) return pool->get(bytes, &p, &cap);
        const cudaError_t e = cudaMalloc(&p, bytes ? bytes : 16);
        cap = bytes;
        return e == cudaSuccess ? nullptr : cudaGetErrorString(e);
    }
    ~DevBlock() {
        if (!p) return;
        cudaStreamSynchronize(st);  // no kernel of this call may still use the block
        if (pool) pool->put(p, cap);
        else cudaFree(p);
    }
};
struct EventPair {
    cudaEvent_t a = nullptr, b = nullptr;
    const char *create() {
        cudaError_t e = cudaEventCreate(&a);
        if (e == cudaSuccess) e = cudaEventCreate(&b);
        return e == cudaSuccess ? nullptr : cudaGetErrorString(e);
    }
    ~EventPair() {
        if (a) cudaEventDestroy(a);
        if (b) cudaEventDestroy(b);
    }
};
}  // namespace cec
