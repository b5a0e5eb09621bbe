// torch_alloc.cpp -- the bf_set_allocator hook pair (include/bf.h) backed by PyTorch's CUDA caching
// allocator, so every device buffer libbf.so allocates (fit work space, forests, staging copies) comes
// from and returns to the same pool as the caller's torch tensors (BASELINE north_star: "PyTorch is used
// only for device memory, streams and process groups").  Built as libbf_torch_alloc.so against the
// installed torch's c10 headers/libraries; plain C entry points, no torch types cross the boundary.
#include <c10/cuda/CUDACachingAllocator.h>
#include <cuda_runtime_api.h>

#include <cstddef>

extern "C" {

// Block of `bytes` on `stream` (the allocator records the stream: the block is reused only in that
// stream's order).  NULL on failure (the library turns it into BF_ENOMEM).
void* bf_torch_alloc(size_t bytes, void* stream, void* /*ctx*/) {
  try {
    return c10::cuda::CUDACachingAllocator::raw_alloc_with_stream(bytes, static_cast<cudaStream_t>(stream));
  } catch (...) {
    return nullptr;
  }
}

void bf_torch_free(void* ptr, void* /*stream*/, void* /*ctx*/) {
  try {
    c10::cuda::CUDACachingAllocator::raw_delete(ptr);
  } catch (...) {
  }
}

}  // extern "C"
