// Test helper (not product, not oracle): NVIDIA's header-only occupancy calculator
// (/usr/local/cuda/include/cuda_occupancy.h), used as an independent pin for the
// oracle's O1 calculator.  Reads lines "T regs smem_static smem_dyn" on stdin and
// prints the CTAs/SM that cudaOccMaxActiveBlocksPerMultiprocessor reports for a
// B200 (cc 10.0) with the given carveout preference (percent; -1 = default) and the
// dynamic-smem opt-in set.  Input lines: "T regs smem_static smem_dyn carveout_pct".
// With the argument "--mask" each output line is "k limitingFactors" (the header's
// OCC_LIMIT_* bits: WARPS 1, REGISTERS 2, SHARED_MEMORY 4, BLOCKS 8).
#include <cuda_occupancy.h>
#include <cstdio>
#include <cstring>

int main(int argc, char **argv) {
    const bool mask = argc > 1 && std::strcmp(argv[1], "--mask") == 0;
    cudaOccDeviceProp prop;
    prop.computeMajor = 10;
    prop.computeMinor = 0;
    prop.maxThreadsPerBlock = 1024;
    prop.maxThreadsPerMultiprocessor = 2048;
    prop.regsPerBlock = 65536;
    prop.regsPerMultiprocessor = 65536;
    prop.warpSize = 32;
    prop.sharedMemPerBlock = 49152;
    prop.sharedMemPerMultiprocessor = 233472;
    prop.numSms = 148;
    prop.sharedMemPerBlockOptin = 232448;
    prop.reservedSharedMemPerBlock = 1024;
    int T, regs, sst, sdyn, pct;
    while (std::scanf("%d %d %d %d %d", &T, &regs, &sst, &sdyn, &pct) == 5) {
        cudaOccFuncAttributes attr;
        attr.maxThreadsPerBlock = 1024;
        attr.numRegs = regs;
        attr.sharedSizeBytes = (size_t)sst;
        attr.partitionedGCConfig = PARTITIONED_GC_OFF;
        attr.shmemLimitConfig = FUNC_SHMEM_LIMIT_OPTIN;
        attr.maxDynamicSharedSizeBytes = 232448 - sst;
        cudaOccDeviceState state;
        state.carveoutConfig = pct;
        state.cacheConfig = CACHE_PREFER_NONE;
        cudaOccResult res;
        cudaOccError e = cudaOccMaxActiveBlocksPerMultiprocessor(&res, &prop, &attr, &state, T, (size_t)sdyn);
        if (mask)
            std::printf("%d %u\n", e == CUDA_OCC_SUCCESS ? res.activeBlocksPerMultiprocessor : -1,
                        e == CUDA_OCC_SUCCESS ? res.limitingFactors : 0u);
        else
            std::printf("%d\n", e == CUDA_OCC_SUCCESS ? res.activeBlocksPerMultiprocessor : -1);
    }
    return 0;
}
