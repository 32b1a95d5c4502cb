// cuda_drv.h -- the CUDA driver API, resolved at run time with dlopen("libcuda.so.1").
//
// liborion links no CUDA runtime and no driver stub, so the library loads (and its
// host-only entry points -- orion_levels, orion_kernel_probe, orion_tuner_replay --
// work) on a machine without a GPU; device entry points return ORION_E_CUDA there.
// The CUstream handles PyTorch hands out are plain driver streams and pass through.
#pragma once
#include <cuda.h>

#include <string>

namespace orion {

// Every driver entry point liborion uses.  Names go through cuda.h's versioning macros
// (cuMemcpyHtoDAsync -> cuMemcpyHtoDAsync_v2, ...), so the member, its type and the
// dlsym'd symbol all refer to the same ABI version.
#define ORION_CU_FUNCS(X)                                                                       \
    X(cuInit) X(cuDeviceGet) X(cuDeviceGetAttribute) X(cuDevicePrimaryCtxRetain)                 \
    X(cuCtxGetCurrent) X(cuCtxSetCurrent) X(cuCtxGetDevice) X(cuModuleLoadData) X(cuModuleUnload) \
    X(cuModuleGetFunction) X(cuFuncGetAttribute) X(cuFuncSetAttribute) X(cuLaunchKernel)          \
    X(cuOccupancyMaxActiveBlocksPerMultiprocessor) X(cuEventCreate) X(cuEventDestroy)             \
    X(cuEventRecord) X(cuEventSynchronize) X(cuEventElapsedTime) X(cuMemcpyHtoDAsync)             \
    X(cuMemcpyDtoHAsync) X(cuStreamSynchronize) X(cuGetErrorString) X(cuGetErrorName)            \
    X(cuMemAlloc) X(cuMemFree) X(cuStreamCreate) X(cuStreamDestroy) X(cuStreamWaitEvent)          \
    X(cuMemsetD32) X(cuMemcpyDtoH) X(cuCtxSynchronize) X(cuEventQuery) X(cuStreamBeginCapture)       \
    X(cuStreamEndCapture) X(cuGraphInstantiate) X(cuGraphLaunch) X(cuGraphExecDestroy) X(cuGraphDestroy) \
    X(cuLaunchKernelEx)

struct Driver {
#define ORION_DECL(f) decltype(&::f) f = nullptr;
    ORION_CU_FUNCS(ORION_DECL)
#undef ORION_DECL
    bool ok = false;
    std::string why;
};

// The process-wide driver table (loaded on first use; thread-safe).
const Driver &drv();

}  // namespace orion
