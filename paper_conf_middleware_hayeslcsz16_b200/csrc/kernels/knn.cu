// knn.cu -- imageDenoising KNN filter (Table 2; math
// per DESIGN.md reading R-O2 = SURVEY §8(c) O2), hand-written for sm_100a.
//
// Per output pixel: 49 window taps, w = 2^(d * (-Noise log2 e) + geo_ij),
// weighted mean, count of w > wthr, SDK lerp toward the centre colour.
//
// Layout: float4 RGBA, row-major, pitch = width.  A CTA of BX x BY threads owns a
// BX-wide, BY*PY-tall output tile; the tile plus a 3-pixel clamp-to-edge halo is
// staged in dynamic shared memory with coalesced float4 loads.  Each thread owns a
// vertical strip of PY pixels and walks the (PY+6) x 7 halo taps once, feeding
// every pixel of its strip that the tap reaches (7*(PY+6) LDS.128 instead of 49*PY).
// Dynamic shared memory = the tile (the kernel's own need); orion_launch may add
// padding on top of it to realise a lower occupancy level.
#include "common.cuh"

#define KNN_R 3
#define KNN_A 49

template <int BX, int BY, int PY>
__device__ __forceinline__ void knn_body(const orion_kargs &a)
{
    constexpr int TW = BX + 2 * KNN_R;
    constexpr int TH = BY * PY + 2 * KNN_R;
    extern __shared__ float4 tile[];
    const int x0 = blockIdx.x * BX;
    const int y0 = a.row_begin + blockIdx.y * (BY * PY);
    load_tile_clamped<TW, TH, BX * BY>(tile, a, x0 - KNN_R, y0 - KNN_R);
    __syncthreads();

    const int tx = threadIdx.x, ty = threadIdx.y;
    const float nl2 = a.fparam[0];
    const float wthr = a.fparam[2];

    float4 c00[PY];
    float ax[PY], ay[PY], az[PY], sw[PY];
    int cnt[PY];
#pragma unroll
    for (int p = 0; p < PY; ++p) {
        c00[p] = tile[(ty * PY + p + KNN_R) * TW + tx + KNN_R];
        ax[p] = ay[p] = az[p] = sw[p] = 0.0f;
        cnt[p] = 0;
    }
#pragma unroll
    for (int r = 0; r < PY + 2 * KNN_R; ++r) {
#pragma unroll
        for (int jj = 0; jj < 2 * KNN_R + 1; ++jj) {
            const float4 c = tile[(ty * PY + r) * TW + tx + jj];
#pragma unroll
            for (int p = 0; p < PY; ++p) {
                const int i = r - KNN_R - p;          // row offset of this tap for pixel p
                if (i < -KNN_R || i > KNN_R) continue; // resolved at compile time
                const int j = jj - KNN_R;
                const float d = dist2(c, c00[p]);
                const float w = ex2(__fmaf_rn(d, nl2, geo_l2_rt(i, j)));
                ax[p] = __fmaf_rn(w, c.x, ax[p]);
                ay[p] = __fmaf_rn(w, c.y, ay[p]);
                az[p] = __fmaf_rn(w, c.z, az[p]);
                sw[p] = __fadd_rn(sw[p], w);
                cnt[p] += (w > wthr);
            }
        }
    }
    const int x = x0 + tx;
    if (x >= a.width) return;
#pragma unroll
    for (int p = 0; p < PY; ++p) {
        const int y = y0 + ty * PY + p;
        if (y < a.row_end) store_out(a, x, y, lerp_out(c00[p], ax[p], ay[p], az[p], sw[p], cnt[p], a));
    }
    fanout_column(a, x, y0 + ty * PY, min(y0 + ty * PY + PY, a.row_end));
}

// T = 128 threads (32 x 4), 16-row tiles.
extern "C" __global__ void __launch_bounds__(128) orion_knn_f4_128(orion_kargs a) { ORION_PROBE(a); knn_body<32, 4, 4>(a); }
// T = 256 threads (32 x 8), 32-row tiles.
extern "C" __global__ void __launch_bounds__(256) orion_knn_f4_256(orion_kargs a) { ORION_PROBE(a); knn_body<32, 8, 4>(a); }
// T = 64 threads (8 x 8), the SDK's CTA shape, 32-row tiles.
extern "C" __global__ void __launch_bounds__(64) orion_knn_f4_64(orion_kargs a) { ORION_PROBE(a); knn_body<8, 8, 4>(a); }
// One pixel per thread (PY = 1): 4x the threads of the strip kernels for the same frame and a
// quarter of the serial tap chain per thread -- small, launch- and latency-bound frames (C1:
// 64 x 64 = 32 CTAs instead of 8).  Same per-pixel tap order, so the same bits.
extern "C" __global__ void __launch_bounds__(128) orion_knn1_f4_128(orion_kargs a) { ORION_PROBE(a); knn_body<32, 4, 1>(a); }
extern "C" __global__ void __launch_bounds__(64) orion_knn1_f4_64(orion_kargs a) { ORION_PROBE(a); knn_body<8, 8, 1>(a); }
