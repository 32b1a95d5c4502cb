// nlm_direct.cuh -- shared body of the direct-form NLM kernels (see nlm_direct.cu).
#pragma once
#include "common.cuh"

#define NLM_R 3
#define NLM_B 3
#define NLM_H (NLM_R + NLM_B)
#define NLM_A 49

template <int BX, int BY, bool REGHEAVY>
__device__ __forceinline__ void nlm_direct_body(const orion_kargs &a)
{
    constexpr int TW = BX + 2 * NLM_H;
    constexpr int TH = BY + 2 * NLM_H;
    extern __shared__ float4 tile[];
    const int x0 = blockIdx.x * BX;
    const int y0 = a.row_begin + blockIdx.y * BY;
    load_tile_clamped<TW, TH, BX * BY>(tile, a, x0 - NLM_H, y0 - NLM_H);
    __syncthreads();

    const int tx = threadIdx.x + NLM_H, ty = threadIdx.y + NLM_H;   // centre in tile coords
    const float nl2 = a.fparam[0];
    const float wthr = a.fparam[2];
    const float4 c00 = tile[ty * TW + tx];

    // the centre patch, negated: each term's (r, g) difference is one FADD2 (fp32x2)
    float4 cp[REGHEAVY ? 2 * NLM_B + 1 : 1][REGHEAVY ? 2 * NLM_B + 1 : 1];
    if (REGHEAVY) {
#pragma unroll
        for (int n = 0; n < 2 * NLM_B + 1; ++n)
#pragma unroll
            for (int m = 0; m < 2 * NLM_B + 1; ++m) {
                const float4 v = tile[(ty + n - NLM_B) * TW + tx + m - NLM_B];
                cp[REGHEAVY ? n : 0][REGHEAVY ? m : 0] = make_float4(-v.x, -v.y, -v.z, 0.0f);
            }
    }

    float ax = 0.f, ay = 0.f, az = 0.f, sw = 0.f;
    int cnt = 0;
#pragma unroll 1
    for (int i = -NLM_R; i <= NLM_R; ++i) {
#pragma unroll (REGHEAVY ? 7 : 1)
        for (int j = -NLM_R; j <= NLM_R; ++j) {
            float d = 0.0f;
#pragma unroll
            for (int n = -NLM_B; n <= NLM_B; ++n) {
#pragma unroll
                for (int m = -NLM_B; m <= NLM_B; ++m) {
                    const float4 s = tile[(ty + i + n) * TW + tx + j + m];
                    float4 nc;
                    if (REGHEAVY) {
                        nc = cp[REGHEAVY ? n + NLM_B : 0][REGHEAVY ? m + NLM_B : 0];
                    } else {
                        const float4 c = tile[(ty + n) * TW + tx + m];
                        nc = make_float4(-c.x, -c.y, -c.z, 0.0f);
                    }
                    // d += dr^2 + dg^2 + db^2, one FFMA per channel (a sum of non-negatives)
                    const float2 e = __fadd2_rn(make_float2(s.x, s.y), make_float2(nc.x, nc.y));
                    const float eb = __fadd_rn(s.z, nc.z);
                    d = __fmaf_rn(eb, eb, __fmaf_rn(e.y, e.y, __fmaf_rn(e.x, e.x, d)));
                }
            }
            const float w = ex2(__fmaf_rn(d, nl2, geo_l2_rt(i, j)));
            const float4 cij = tile[(ty + i) * TW + tx + j];
            ax = __fmaf_rn(w, cij.x, ax);
            ay = __fmaf_rn(w, cij.y, ay);
            az = __fmaf_rn(w, cij.z, az);
            sw = __fadd_rn(sw, w);
            cnt += (w > wthr);
        }
    }
    const int x = x0 + threadIdx.x, y = y0 + threadIdx.y;
    if (x < a.width && y < a.row_end)
        ((float4 *)a.dst)[frame_px(a) + (size_t)(y - a.dst_row_begin) * (size_t)a.width + x] =
            lerp_out(c00, ax, ay, az, sw, cnt, a);
}

