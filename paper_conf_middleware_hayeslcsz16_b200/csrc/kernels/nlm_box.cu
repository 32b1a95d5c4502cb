// nlm_box.cu -- imageDenoising NLM filter, separable box-sum form (the hot kernel of
// configs C2 / C5).  Same result as the direct definition (
// math per DESIGN.md reading R-O2) up to the order of the patch summation:
//
//   D_o(x,y) = sum_{n,m=-3..3} d_o(x+m, y+n),   d_o(u,v) = |p(u+j, v+i) - p(u,v)|^2
//
// is a 7x7 box sum of the per-offset difference image d_o, so it is evaluated as
// vertical 7-sums C_o(u,y) = sum_n d_o(u, y+n) followed by horizontal 7-sums
// D_o(x,y) = sum_m C_o(x+m, y): ~2 difference evaluations per pixel and offset
// instead of 49 (DESIGN.md §"nlm_f4": 2401 -> ~70 patch terms per pixel).
//
// CTA = 128 threads, output tile TW = 120 columns x TH = 16 rows.  The input tile
// (TW+12) x (TH+12) pixels with a 6-pixel clamp-to-edge halo is staged once in
// shared memory as three planar fp32 arrays (r, g, b: conflict-free LDS.32, no
// wasted alpha bytes).  Per window offset o (49 of them):
//   phase A: thread u (0..125) walks column x0-3+u downward, forms d_o for the TH+6
//            rows it needs and writes the TH vertical 7-sums C_o(u, .) to smem;
//   phase B: thread (g, rg) owns 4 strided columns g + 30k and TH/4 rows; per pixel it
//            reads the 7 C values of the row (conflict-free LDS.32), forms D_o, the
//            weight w = 2^(D_o * (-Noise log2 e) + geo_o), and accumulates w*p, w,
//            [w > wthr].
// Two __syncthreads per offset separate the phases.
#include "common.cuh"

#define BOX_R 3
#define BOX_B 3
#define BOX_HALO (BOX_R + BOX_B)

template <int TW, int TH, int NT>
__device__ __forceinline__ void nlm_box_body(const orion_kargs &a)
{
    constexpr int NC = 4;                       // columns per thread in phase B
    static_assert(TW % NC == 0, "column groups");
    constexpr int PW = TW + 2 * BOX_HALO;       // planar tile width  (x0-6 .. x0+TW+6)
    constexpr int PH = TH + 2 * BOX_HALO;       // planar tile height (y0-6 .. y0+TH+6)
    constexpr int CW = TW + 2 * BOX_B;          // columns of C (x0-3 .. x0+TW+3)
    constexpr int CP = CW + 2;                  // C row pitch (floats)
    constexpr int NG = TW / NC;                 // column groups in phase B
    constexpr int RPT = TH / 4;                 // rows per thread in phase B (4 row groups)
    static_assert(NG * (TH / RPT) <= NT && CW <= NT, "thread mapping");
    extern __shared__ float4 smem4[];
    float *pr = reinterpret_cast<float *>(smem4);
    float *pg = pr + PW * PH;
    float *pb = pg + PW * PH;
    float *cs = pb + PW * PH;                   // C_o: TH rows x CP

    const int tid = threadIdx.x;
    const int x0 = blockIdx.x * TW;
    const int y0 = a.row_begin + blockIdx.y * TH;
    {   // stage the planar tile (coalesced float4 loads, clamp-to-edge in global coords)
        const float4 *src = (const float4 *)a.src;
        for (int idx = tid; idx < PW * PH; idx += NT) {
            const int ty = idx / PW, tx = idx - ty * PW;
            const int gx = clampi(x0 - BOX_HALO + tx, 0, a.width - 1);
            const int gy = clampi(y0 - BOX_HALO + ty, 0, a.height - 1);
            const float4 v = __ldg(src + (size_t)(gy - a.src_row_begin) * (size_t)a.width + gx);
            pr[idx] = v.x;
            pg[idx] = v.y;
            pb[idx] = v.z;
        }
    }
    __syncthreads();

    const float nl2 = a.fparam[0];
    const float wthr = a.fparam[2];
    // phase B ownership: column group g owns the NC strided columns g, g+NG, g+2NG, ..
    // (consecutive lanes -> consecutive shared-memory words: conflict-free LDS.32),
    // row group rg owns RPT consecutive rows.
    const int g = tid % NG, rg = tid / NG;
    const bool ownB = tid < NG * (TH / RPT);
    const int by = rg * RPT;
    float ax[RPT][NC], ay[RPT][NC], az[RPT][NC], sw[RPT][NC];
    int cnt[RPT][NC];
#pragma unroll
    for (int r = 0; r < RPT; ++r)
#pragma unroll
        for (int k = 0; k < NC; ++k) {
            ax[r][k] = ay[r][k] = az[r][k] = sw[r][k] = 0.0f;
            cnt[r][k] = 0;
        }

#pragma unroll 1
    for (int o = 0; o < 49; ++o) {
        const int i = o / 7 - BOX_R, j = o % 7 - BOX_R;
        // ---- phase A: vertical 7-sums of d_o down column u ------------------------------
        if (tid < CW) {
            const int cu = tid + BOX_B;          // planar column of x0-3+tid
            float dwin[TH + 2 * BOX_B];
#pragma unroll
            for (int r = 0; r < TH + 2 * BOX_B; ++r) {   // rows y0-3+r
                const int pc = (r + BOX_B) * PW + cu;     // p(u, v)
                const int ps = pc + i * PW + j;           // p(u+j, v+i)
                const float dx = __fsub_rn(pr[ps], pr[pc]);
                const float dy = __fsub_rn(pg[ps], pg[pc]);
                const float dz = __fsub_rn(pb[ps], pb[pc]);
                dwin[r] = __fmaf_rn(dz, dz, __fmaf_rn(dy, dy, __fmul_rn(dx, dx)));
            }
#pragma unroll
            for (int y = 0; y < TH; ++y) {
                float s = dwin[y];
#pragma unroll
                for (int n = 1; n < 2 * BOX_B + 1; ++n) s = __fadd_rn(s, dwin[y + n]);
                cs[y * CP + tid] = s;
            }
        }
        __syncthreads();
        // ---- phase B: horizontal 7-sums, weights, accumulation --------------------------
        if (ownB) {
            const float geo = geo_l2_rt(i, j);
#pragma unroll
            for (int r = 0; r < RPT; ++r) {
                const float *crow = cs + (by + r) * CP;
                const int prow = (by + r + BOX_HALO + i) * PW + BOX_HALO + j;
#pragma unroll
                for (int k = 0; k < NC; ++k) {
                    const int xl = g + k * NG;
                    float D = crow[xl];
#pragma unroll
                    for (int m = 1; m < 2 * BOX_B + 1; ++m) D = __fadd_rn(D, crow[xl + m]);
                    const float w = exp2f(__fmaf_rn(D, nl2, geo));
                    ax[r][k] = __fmaf_rn(w, pr[prow + xl], ax[r][k]);
                    ay[r][k] = __fmaf_rn(w, pg[prow + xl], ay[r][k]);
                    az[r][k] = __fmaf_rn(w, pb[prow + xl], az[r][k]);
                    sw[r][k] = __fadd_rn(sw[r][k], w);
                    cnt[r][k] += (w > wthr);
                }
            }
        }
        __syncthreads();
    }
    if (!ownB) return;
    float4 *dst = (float4 *)a.dst;
#pragma unroll
    for (int r = 0; r < RPT; ++r) {
        const int y = y0 + by + r;
        if (y >= a.row_end) break;
#pragma unroll
        for (int k = 0; k < NC; ++k) {
            const int xl = g + k * NG;
            const int x = x0 + xl;
            if (x >= a.width) continue;
            const int pc = (by + r + BOX_HALO) * PW + xl + BOX_HALO;
            const float4 c00 = make_float4(pr[pc], pg[pc], pb[pc], 0.0f);
            dst[(size_t)(y - a.dst_row_begin) * (size_t)a.width + x] =
                lerp_out(c00, ax[r][k], ay[r][k], az[r][k], sw[r][k], cnt[r][k], a);
        }
    }
}

// Shared memory: 3 planar (TW+12)x(TH+12) fp32 planes + TH x CP floats of C.
extern "C" __global__ void __launch_bounds__(128) orion_nlm_box_f4_128(orion_kargs a)
{
    nlm_box_body<120, 16, 128>(a);
}
