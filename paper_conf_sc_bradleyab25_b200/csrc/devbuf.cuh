// devbuf.cuh -- stream-ordered device allocations with RAII + error macros.
#pragma once
#include <cuda_runtime.h>
#include "internal.h"

#define FSGC_CUDA(call)                                                              \
    do {                                                                             \
        cudaError_t e_ = (call);                                                     \
        if (e_ != cudaSuccess) {                                                     \
            fsgc_set_error("%s failed: %s (%s:%d)", #call, cudaGetErrorString(e_),   \
                           __FILE__, __LINE__);                                      \
            return e_ == cudaErrorMemoryAllocation ? FSGC_ERR_OOM : FSGC_ERR_CUDA;   \
        }                                                                            \
    } while (0)

// the library's own stream-ordered memory pool on the current device
// (graph.cu): load temporaries are cached there, not in the device's default
// pool, so the host application's allocators are not affected
cudaMemPool_t fsgc_device_pool();

template <typename T>
struct DevBuf {
    T* ptr = nullptr;
    size_t count = 0;
    cudaStream_t stream = nullptr;
    DevBuf() = default;
    DevBuf(const DevBuf&) = delete;
    DevBuf& operator=(const DevBuf&) = delete;
    ~DevBuf() { release(); }
    cudaError_t alloc(size_t n, cudaStream_t s) {
        release();
        stream = s;
        count = n;
        if (n == 0) return cudaSuccess;
        cudaMemPool_t pool = fsgc_device_pool();
        if (!pool) return cudaErrorInitializationError;
        return cudaMallocFromPoolAsync((void**)&ptr, n * sizeof(T), pool, s);
    }
    void release() {
        if (ptr) cudaFreeAsync(ptr, stream);
        ptr = nullptr;
        count = 0;
    }
    T* take() {  // transfer ownership out
        T* p = ptr;
        ptr = nullptr;
        count = 0;
        return p;
    }
};
