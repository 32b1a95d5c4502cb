// common.cuh -- helpers shared by the Orion sm_100a kernels (product code).
//
// Every kernel is compiled ONCE to PTX (nvcc -arch=compute_100a -fmad=false) and
// then assembled by liborion once per register cap (orion_build_variants), so the
// value path must not depend on ptxas' register allocation: all floating-point
// arithmetic is explicit (.rn mul/add/fma, no contraction freedom) and therefore
// bit-identical across every occupancy variant (SURVEY §7 hard part 2).
#pragma once
#include <stdint.h>
#include "../orion_kargs.h"

#define ORION_DEVICE __device__ __forceinline__

// Residency probe (build time only, a.probe != NULL): thread 0 of each CTA counts the CTAs
// resident on its SM (probe[smid]), records the maximum (probe[1024 + smid]) and holds the
// CTA -- all its warps waiting at a barrier, with the function's real registers and shared
// memory allocated -- for 20 us; the kernel then returns without touching its buffers.  orion_build_variants launches a full
// grid this way to MEASURE the CTAs/SM each occupancy variant actually gets.
ORION_DEVICE bool orion_probe(const orion_kargs &a)
{
    // programmatic dependent launch (orion_launch with ORION_PDL=1): let the stream's next grid
    // be scheduled now, and wait here until the previous grid has completed and its memory is
    // visible -- before any load -- unless the caller asserted the launch independent of it
    // (ORION_ARGS_INDEPENDENT: the CTAs start in the previous grid's last wave).  Both are no-ops
    // for a normal launch.
    if (!a.dep_late) asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    if (!a.nowait) asm volatile("griddepcontrol.wait;" ::: "memory");
    if (a.probe == nullptr) return false;
    if (threadIdx.x == 0 && threadIdx.y == 0) {
        unsigned smid;
        asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
        smid &= 1023u;
        const unsigned c = atomicAdd(a.probe + smid, 1u) + 1u;
        atomicMax(a.probe + 1024 + smid, c);
        unsigned long long t0, t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
        do {
            asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        } while (t - t0 < 20000ull);
        atomicSub(a.probe + smid, 1u);
    }
    __syncthreads();   // every warp stays resident (registers are granted per warp) until then
    return true;
}
#define ORION_PROBE(a) \
    if (orion_probe(a)) return

// ---- orion_chain: tile-level dependencies between consecutive launches -------------------------
// A chained launch (orion.h orion_chain) does not wait for the whole previous grid: its CTA at
// tile (bx, by) waits only until the previous launch of the chain has completed the tiles whose
// output it reads or whose input it overwrites -- the 3 x 3 neighbourhood (the stencil halos are
// smaller than a tile) plus an optional extra rectangle (SRAD: the ROI tiles that write the
// statistics slots) -- and publishes its own completion at the end.  Flags hold the epoch of the
// last launch that completed the tile: wait for >= epoch-1, publish epoch (release / acquire at
// GPU scope; the data written by other SMs is then read through L2: cp.async.cg / ld.global.cg).
ORION_DEVICE unsigned chain_ld_acquire(const unsigned *p)
{
    unsigned v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
ORION_DEVICE void chain_wait_tile(const orion_kargs &a, int x, int y, unsigned long long t0)
{
    const unsigned *f = a.chain + (size_t)y * gridDim.x + x;
    const unsigned need = a.chain_epoch - 1u;
    while (chain_ld_acquire(f) < need) {
        __nanosleep(200);
        unsigned long long t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        if (t - t0 > 4000000000ull) __trap();   // 4 s: a broken chain (misuse) fails loudly, never hangs
    }
}
// Called by every thread of the CTA (contains a barrier).  ex0 > ex1: no extra rectangle.  The
// lanes of warp 0 poll one tile each (k < 9: the 3 x 3 neighbourhood, then the extra rectangle),
// so a CTA pays one flag round trip, not one per tile.
ORION_DEVICE void chain_wait(const orion_kargs &a, int ex0, int ex1, int ey0, int ey1)
{
    if (threadIdx.y == 0) {
        unsigned long long t0;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
        const int gx = gridDim.x, gy = gridDim.y;
        const int ew = ex1 >= ex0 ? ex1 - ex0 + 1 : 0, eh = ey1 >= ey0 ? ey1 - ey0 + 1 : 0;
        for (int k = threadIdx.x; k < 9 + ew * eh; k += 32) {
            int x, y;
            if (k < 9) {
                x = (int)blockIdx.x + k % 3 - 1;
                y = (int)blockIdx.y + k / 3 - 1;
            } else {
                x = ex0 + (k - 9) % ew;
                y = ey0 + (k - 9) / ew;
            }
            if (x >= 0 && x < gx && y >= 0 && y < gy) chain_wait_tile(a, x, y, t0);
        }
        __syncwarp();
    }
    __syncthreads();
}
// Called by every thread of the CTA after its last global access (contains a barrier).
ORION_DEVICE void chain_signal(const orion_kargs &a)
{
    __syncthreads();
    if (threadIdx.x == 0 && threadIdx.y == 0) {
        __threadfence();
        unsigned *f = a.chain + (size_t)blockIdx.y * gridDim.x + blockIdx.x;
        asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(f), "r"(a.chain_epoch) : "memory");
    }
}

ORION_DEVICE int clampi(int v, int lo, int hi) { return v < lo ? lo : (v > hi ? hi : v); }

// Frame of a batched denoiser launch (orion_args.batch: gridDim.z whole width x height frames
// stacked in src / dst): the pixel offset of this CTA's frame (0 for a single frame).
ORION_DEVICE size_t frame_px(const orion_kargs &a)
{
    return (size_t)blockIdx.z * (size_t)a.width * (size_t)a.height;
}

// Row of the input slab a staged tile reads for global row gy: clamp-to-edge in GLOBAL
// coordinates (the definition), then into the rows the slab holds.  The second clamp never
// changes a row that a stored output depends on (the host guarantees the slab covers
// [row_begin - halo, row_end + halo) after global clamping); it only keeps the tile rows past
// row_end -- computed, never stored -- inside the slab's allocation (a band whose height is
// not a multiple of the tile height would otherwise read up to TH - 1 rows past it).
ORION_DEVICE int slab_row(const orion_kargs &a, int gy)
{
    return clampi(clampi(gy, 0, a.height - 1), a.src_row_begin, a.src_row_end - 1);
}

// Squared RGB distance, |a - b|^2 with a fixed operation order.
ORION_DEVICE float dist2(float4 a, float4 b)
{
    float dx = __fsub_rn(a.x, b.x), dy = __fsub_rn(a.y, b.y), dz = __fsub_rn(a.z, b.z);
    return __fmaf_rn(dz, dz, __fmaf_rn(dy, dy, __fmul_rn(dx, dx)));
}

// Cooperative, coalesced load of a TW x TH float4 tile whose top-left corner is
// global pixel (gx0, gy0), with clamp-to-edge addressing in GLOBAL coordinates
// (so a row-sharded launch reads exactly what the full-image launch reads).
template <int TW, int TH, int NT>
ORION_DEVICE void load_tile_clamped(float4 *tile, const orion_kargs &a, int gx0, int gy0)
{
    const float4 *src = (const float4 *)a.src + frame_px(a);
    const int W = a.width;
    const int tid = threadIdx.y * blockDim.x + threadIdx.x;
    for (int idx = tid; idx < TW * TH; idx += NT) {
        int ty = idx / TW;
        int tx = idx - ty * TW;
        int gx = clampi(gx0 + tx, 0, W - 1);
        int gy = slab_row(a, gy0 + ty);
        tile[idx] = __ldg(src + (size_t)(gy - a.src_row_begin) * (size_t)W + gx);
    }
}

// cp.async (LDGSTS) of 8 / 4 bytes global -> shared: no registers, every copy of a thread in
// flight at once (one memory latency for a whole staged tile instead of one per unrolled
// batch of register loads).  Completed by cp_async_wait_all() + a barrier.
ORION_DEVICE void cpa8(void *sdst, const void *gsrc)
{
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8;\n" ::"r"((unsigned)__cvta_generic_to_shared(sdst)),
                 "l"(gsrc) : "memory");
}
ORION_DEVICE void cpa4(void *sdst, const void *gsrc)
{
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;\n" ::"r"((unsigned)__cvta_generic_to_shared(sdst)),
                 "l"(gsrc) : "memory");
}
ORION_DEVICE void cpa16(void *sdst, const void *gsrc)
{
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"((unsigned)__cvta_generic_to_shared(sdst)),
                 "l"(gsrc) : "memory");
}
ORION_DEVICE void cp_async_wait_all() { asm volatile("cp.async.wait_all;\n" ::: "memory"); }

// Output pixel (x, y) (global row y) into dst (rows from dst_row_begin).
ORION_DEVICE void store_out(const orion_kargs &a, int x, int y, float4 o)
{
    ((float4 *)a.dst)[frame_px(a) + (size_t)(y - a.dst_row_begin) * (size_t)a.width + x] = o;
}

// Fan-out of this thread's output column x, rows [y0, y1) (already in dst, written by this
// same thread): copied into every fan-out image (full images, row y at y * width) -- the
// gather of a row-sharded frame written straight into each rank's buffer over NVLink peer
// memory (C5) as each tile completes.  A compact rolled loop after the unrolled epilogue, so
// the kernel's hot code does not grow when fan-out is used.
ORION_DEVICE void fanout_column(const orion_kargs &a, int x, int y0, int y1)
{
    if (a.nfan == 0) return;
    const float4 *src = (const float4 *)a.dst + (size_t)(y0 - a.dst_row_begin) * (size_t)a.width + x;
#pragma unroll 1
    for (int y = y0; y < y1; ++y, src += a.width) {
        const float4 o = *src;
#pragma unroll 1
        for (int f = 0; f < a.nfan; ++f) ((float4 *)a.fan[f])[(size_t)y * (size_t)a.width + x] = o;
    }
}

// Final SDK imageDenoising blend: clr = acc/sw; out = clr + (c00 - clr) * q.
ORION_DEVICE float4 lerp_out(float4 c00, float ax, float ay, float az, float sw, int cnt,
                             const orion_kargs &a)
{
    const float lerpc = a.fparam[1];
    const float q = (cnt >= a.iparam0) ? lerpc : __fsub_rn(1.0f, lerpc);
    // acc / sw as acc * (1/sw) with one MUFU reciprocal (rcp.approx, <= 1 ulp): sw >= 1 always
    // (the centre weight is exactly 1), so the quotient is within 2 ulp of the IEEE division
    // -- far inside the 1e-5 tolerance -- and the epilogue needs no division subroutine.
    float rs;
    asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(rs) : "f"(sw));
    float cx = __fmul_rn(ax, rs), cy = __fmul_rn(ay, rs), cz = __fmul_rn(az, rs);
    float4 o;
    o.x = __fmaf_rn(__fsub_rn(c00.x, cx), q, cx);
    o.y = __fmaf_rn(__fsub_rn(c00.y, cy), q, cy);
    o.z = __fmaf_rn(__fsub_rn(c00.z, cz), q, cz);
    o.w = 0.0f;
    return o;
}


// 2^x on the SFU (MUFU.EX2, ~2 ulp), flushing sub-normal results to zero: the weights
// that small (< 2^-126) are below every threshold and vanish in the weight sums, which
// always hold the centre weight 1.  Saves exp2f's sub-normal rescaling (FSETP + 2 FMUL).
ORION_DEVICE float ex2(float x)
{
    float y;
    asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}

// Same term evaluated at run time: (i*i + j*j) * (-log2(e)/49) with one rounding.
ORION_DEVICE float geo_l2_rt(int i, int j)
{
    return __fmul_rn((float)(i * i + j * j), (float)(-1.4426950408889634 / 49.0));
}
