// Entries for tools/tmem_occupancy_probe.py: a plain kernel and three that allocate 32 / 128 / 512
// tensor-memory columns (alloc, relinquish, dealloc).
extern "C" __global__ void __launch_bounds__(32) k_plain(unsigned *o) { o[threadIdx.x] = threadIdx.x; }
template <int C>
__device__ void body(unsigned *o) {
    __shared__ unsigned base;
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" :: "r"((unsigned)__cvta_generic_to_shared(&base)), "n"(C) : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncwarp();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    o[threadIdx.x] = base;
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" :: "r"(base), "n"(C) : "memory");
}
extern "C" __global__ void __launch_bounds__(32) k_tm32(unsigned *o) { body<32>(o); }
extern "C" __global__ void __launch_bounds__(32) k_tm128(unsigned *o) { body<128>(o); }
extern "C" __global__ void __launch_bounds__(32) k_tm512(unsigned *o) { body<512>(o); }
