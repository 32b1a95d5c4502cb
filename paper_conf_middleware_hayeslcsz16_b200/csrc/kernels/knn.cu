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

// The exponent of a tap's weight, w = 2^e: e = d * (-Noise log2 e) + geo_ij with d = |c - c00|^2 =
// (dr^2 + dg^2) + db^2 -- the (r, g) difference and squares packed (FADD2, FMUL2), a sum of
// non-negative terms 3 roundings deep (reading R-NLM-FP).  nrg / nb: the negated centre colour.
ORION_DEVICE float knn_tap_exponent(float4 c, float2 nrg, float nb, float nl2, float geo)
{
    const float2 drg = __fadd2_rn(make_float2(c.x, c.y), nrg);
    const float2 q = __fmul2_rn(drg, drg);
    const float db = __fadd_rn(c.z, nb);
    const float d = __fmaf_rn(db, db, __fadd_rn(q.x, q.y));
    return __fmaf_rn(d, nl2, geo);
}

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

    const float ethr = a.fparam[3];          // log2(wthr): [w > wthr] decided on the exponent

    // packed fp32x2 taps (FADD2 / FMUL2 / FFMA2, two IEEE .rn operations each): the (r, g)
    // difference, its squares, and the accumulations (w r, w g) and (w b, w) in pairs
    float2 nrg[PY];                          // -(r, g) of the centre pixel (the centre itself is
    float nb[PY];                            //  read again from the tile for the blend)
    float2 axy[PY], azs[PY];                 // (sum w r, sum w g), (sum w b, sum w)
    int cnt[PY];
#pragma unroll
    for (int p = 0; p < PY; ++p) {
        const float4 c00 = tile[(ty * PY + p + KNN_R) * TW + tx + KNN_R];
        nrg[p] = make_float2(-c00.x, -c00.y);
        nb[p] = -c00.z;
        axy[p] = azs[p] = make_float2(0.0f, 0.0f);
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
                const float e = knn_tap_exponent(c, nrg[p], nb[p], nl2, geo_l2_rt(i, j));
                const float w = ex2(e);
                axy[p] = __ffma2_rn(make_float2(w, w), make_float2(c.x, c.y), axy[p]);
                azs[p] = __ffma2_rn(make_float2(w, w), make_float2(c.z, 1.0f), azs[p]);
                cnt[p] += (e > ethr);
            }
        }
    }
    const int x = x0 + tx;
    if (x >= a.width) return;
#pragma unroll
    for (int p = 0; p < PY; ++p) {
        const int y = y0 + ty * PY + p;
        const float4 c00 = tile[(ty * PY + p + KNN_R) * TW + tx + KNN_R];
        if (y < a.row_end) store_out(a, x, y, lerp_out(c00, axy[p].x, axy[p].y, azs[p].x, azs[p].y, cnt[p], a));
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

// ---- tap-split form (knn_f4_t16): 16 threads per pixel -----------------------------------------
// Small frames (C1: 64 x 64 = 4096 pixels) are latency-bound: one pixel per thread still walks
// a serial chain of 49 taps on 32 of 148 SMs.  Here the 49 taps of a pixel are split over the LP
// lanes of a lane group (lane g takes taps k = g, g+LP, ..., k -> (i, j) = (k/7 - 3, k%7 - 3)),
// read straight from global memory (clamp-to-edge in global coordinates; the frame is L1 / L2
// resident), and the LP partial sums are combined by a fixed xor-shuffle tree whose result lane
// 0 of the group writes.  Every weight is computed exactly as in knn_body (same tap arithmetic),
// so the counts -- hence the lerp branch -- are the same; only the order of the weighted sums
// differs (within the 1e-5 tolerance; bit-identical across occupancy levels, which share this
// code).  CTA = 128 threads = 128 / LP pixels of one row.  (LP = 8, round 1's knn_f4_t8, measured
// 3.4-3.6 vs 3.0-3.07 us per C1 frame and removed.)
template <int LP>
__device__ __forceinline__ void knn_tap_split_body(const orion_kargs &a)
{
    static_assert(LP == 8 || LP == 16, "lanes per pixel: a power of two dividing 32");
    const int g = threadIdx.x & (LP - 1);
    const int x = blockIdx.x * (128 / LP) + (threadIdx.x / LP);
    const int y = a.row_begin + blockIdx.y;
    const int W = a.width, H = a.height;
    const int xc = min(x, W - 1);
    const float4 *src = (const float4 *)a.src + frame_px(a) - (size_t)a.src_row_begin * (size_t)W;
    const float nl2 = a.fparam[0];
    const float4 c00 = __ldg(src + (size_t)y * (size_t)W + xc);
    const float2 nrg = make_float2(-c00.x, -c00.y);
    const float nb = -c00.z;
    const float ethr = a.fparam[3];
    float ax = 0.0f, ay = 0.0f, az = 0.0f, sw = 0.0f;
    int cnt = 0;
#pragma unroll
    for (int s = 0; s < (KNN_A + LP - 1) / LP; ++s) {
        const int k = g + LP * s;
        if (k >= KNN_A) break;                     // only lane 0 of a group has the last tap (k = 48)
        const int i = k / 7 - KNN_R, j = k % 7 - KNN_R;
        const int gy = clampi(y + i, 0, H - 1), gx = clampi(xc + j, 0, W - 1);
        const float4 c = __ldg(src + (size_t)gy * (size_t)W + gx);
        const float e = knn_tap_exponent(c, nrg, nb, nl2, geo_l2_rt(i, j));
        const float w = ex2(e);
        ax = __fmaf_rn(w, c.x, ax);
        ay = __fmaf_rn(w, c.y, ay);
        az = __fmaf_rn(w, c.z, az);
        sw = __fadd_rn(sw, w);
        cnt += (e > ethr);
    }
#pragma unroll
    for (int o = LP / 2; o > 0; o >>= 1) {
        ax = __fadd_rn(ax, __shfl_xor_sync(0xffffffffu, ax, o));
        ay = __fadd_rn(ay, __shfl_xor_sync(0xffffffffu, ay, o));
        az = __fadd_rn(az, __shfl_xor_sync(0xffffffffu, az, o));
        sw = __fadd_rn(sw, __shfl_xor_sync(0xffffffffu, sw, o));
        cnt += __shfl_xor_sync(0xffffffffu, cnt, o);
    }
    if (g == 0 && x < W) {
        store_out(a, x, y, lerp_out(c00, ax, ay, az, sw, cnt, a));
        fanout_column(a, x, y, y + 1);
    }
}
// 16 lanes per pixel (3-4 taps each), 8 pixels of one row per CTA.
extern "C" __global__ void __launch_bounds__(128) orion_knn16_f4_128(orion_kargs a) { ORION_PROBE(a); knn_tap_split_body<16>(a); }
