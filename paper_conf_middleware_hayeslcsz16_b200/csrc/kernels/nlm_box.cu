// nlm_box.cu -- imageDenoising NLM filter, separable box-sum form with symmetric
// offset pairs: the hot kernel of configs C2 / C5.  Same result as the direct
// definition (PAPER.md; math per DESIGN.md reading R-O2) up to the order of
// the patch summation:
//
//   D_o(x,y) = sum_{n,m=-3..3} d_o(x+m, y+n),   d_o(u,v) = |p(u+j, v+i) - p(u,v)|^2
//
// (1) D_o is a 7x7 box sum of the difference image d_o: horizontal 7-sums
//     H_o(u,v) = sum_m d_o(u+m, v), then vertical 7-sums D_o(x,y) = sum_n H_o(x, y+n).
// (2) d_{-o}(u,v) = d_o(u-j, v-i), hence D_{-o}(x,y) = D_o(x-j, y-i): one box sum serves
//     the offset pair (o, -o).  The 48 non-centre offsets form 24 pairs; the centre
//     offset has D = 0, w = 1 exactly.
// Both are exact identities; only the order of the fp32 additions differs from the
// definition (every partial sum is a sum of non-negative terms, at most 4 roundings
// deep: see DESIGN.md §nlm_f4 for the error budget against the 1e-5 tolerance).
//
// CTA = 128 threads (4 warps); output tile TW = 122 columns x TH = 23 rows.
// Shared memory: the input tile (TW+18) x (TH+12) with a 9-column / 6-row
// clamp-to-edge halo as three planar fp32 arrays (odd pitch), and one H_o buffer of
// 32 rows x 128 columns (odd pitch).  Per offset pair:
//   phase A: warp w computes H_o for columns [32w, 32w+32) of the H buffer; lane = row
//            (32 rows = TH + 9), sliding along the row over 38 difference values.
//            Lanes touch 32 different rows of an odd-pitch array: conflict-free.
//   phase B: thread t owns output column x0+t and all TH rows: vertical 7-sums of
//            H_o down column t+3 give D_o(x, .), and down column t+3-j, shifted by -i
//            rows, give D_{-o}(x, .); weights w = 2^(D * (-Noise log2 e) + geo) and
//            the accumulation of w*p, w and [w > wthr] for both offsets.  Lanes touch
//            consecutive columns: conflict-free.
// Two __syncthreads per pair.  ~4 LDS per pixel-offset in phase B, ~0.9 difference
// evaluations per pixel-offset in phase A (vs 49 patch terms in the direct form).
#include "common.cuh"

#define PB_R 3   // window radius
#define PB_B 3   // patch radius

namespace {

constexpr int TW = 122, TH = 23, NT = 128;
constexpr int AR = TH + 9;                  // phase-A rows (H rows): y0-6 .. y0+TH+3
constexpr int HC = TW + 6;                  // H columns: x0-3 .. x0+TW+3
constexpr int HP = HC + 1;                  // odd H pitch
constexpr int PC = TW + 18;                 // image tile columns: x0-9 .. x0+TW+9
constexpr int PR = TH + 12;                 // image tile rows:    y0-6 .. y0+TH+6
constexpr int PW = PC + 1;                  // odd plane pitch
static_assert(AR == 32 && HC == 4 * 32 && NT == 128, "phase A: one lane per row, one warp per 32 H columns");
static_assert(TW <= NT, "phase B: one thread per output column");

// Blocked 7-term window sums of a[0 .. N+5]: out[k] = a[k] + ... + a[k+6] evaluated as
// ((a[k]+a[k+1]) + (a[k+2]+a[k+3])) + ((a[k+4]+a[k+5]) + a[k+6]) -- 4 additions per
// output with the pair sums shared; every partial sum is a sum of non-negatives.
template <int N>
ORION_DEVICE void window7(const float (&a)[N + 6], float (&out)[N])
{
    float p[N + 5];
#pragma unroll
    for (int k = 0; k < N + 5; ++k) p[k] = __fadd_rn(a[k], a[k + 1]);
#pragma unroll
    for (int k = 0; k < N; ++k)
        out[k] = __fadd_rn(__fadd_rn(p[k], p[k + 2]), __fadd_rn(p[k + 4], a[k + 6]));
}

}  // namespace

extern "C" __global__ void __launch_bounds__(128) orion_nlm_box_f4_128(orion_kargs a)
{
    extern __shared__ float4 smem4[];
    float *pr = reinterpret_cast<float *>(smem4);
    float *pg = pr + PR * PW;
    float *pb = pg + PR * PW;
    float *hs = pb + PR * PW;               // H_o: AR rows x HP

    const int tid = threadIdx.x;
    const int lane = tid & 31, warp = tid >> 5;
    const int x0 = blockIdx.x * TW;
    const int y0 = a.row_begin + blockIdx.y * TH;
    {   // stage the planar tile (coalesced float4 loads, clamp-to-edge in global coords)
        const float4 *src = (const float4 *)a.src;
        for (int idx = tid; idx < PC * PR; idx += NT) {
            const int ty = idx / PC, tx = idx - ty * PC;
            const int gx = clampi(x0 - 9 + tx, 0, a.width - 1);
            const int gy = clampi(y0 - 6 + ty, 0, a.height - 1);
            const float4 v = __ldg(src + (size_t)(gy - a.src_row_begin) * (size_t)a.width + gx);
            pr[ty * PW + tx] = v.x;
            pg[ty * PW + tx] = v.y;
            pb[ty * PW + tx] = v.z;
        }
    }
    __syncthreads();

    const float nl2 = a.fparam[0];
    const float wthr = a.fparam[2];
    // phase-B state: column t, rows 0..TH-1.  Counts are packed 4 x 8 bits per word (<= 49).
    const int t = tid;
    float ax[TH], ay[TH], az[TH], sw[TH];
    unsigned cnt[(TH + 3) / 4];
    {
        const unsigned c1 = (1.0f > wthr) ? 1u : 0u;   // centre offset: D = 0, w = 1 exactly
#pragma unroll
        for (int r = 0; r < TH; ++r) {
            const int pc = (r + 6) * PW + t + 9;
            ax[r] = pr[pc];
            ay[r] = pg[pc];
            az[r] = pb[pc];
            sw[r] = 1.0f;
        }
#pragma unroll
        for (int q = 0; q < (TH + 3) / 4; ++q) cnt[q] = c1 * 0x01010101u;
    }

#pragma unroll 1
    for (int pi = 0; pi < 24; ++pi) {
        // half-plane pair representative o = (i, j): (0,1..3) then (1..3, -3..3)
        const int i = pi < 3 ? 0 : (pi - 3) / 7 + 1;
        const int j = pi < 3 ? pi + 1 : (pi - 3) % 7 - 3;
        // ---- phase A: H_o(u, v) for this warp's 32 columns, lane = row -------------------
        {
            const int r = lane;                           // tile row of v (y0-6+r)
            const int cb = 3 + 32 * warp;                 // tile column of u for the first d
            const float *cr = pr + r * PW + cb, *cg = pg + r * PW + cb, *cbp = pb + r * PW + cb;
            const int so = i * PW + j;                    // shift to p(u+j, v+i)
            float d[38];
#pragma unroll
            for (int q = 0; q < 38; ++q) {
                const float dx = __fsub_rn(cr[q + so], cr[q]);
                const float dy = __fsub_rn(cg[q + so], cg[q]);
                const float dz = __fsub_rn(cbp[q + so], cbp[q]);
                d[q] = __fmaf_rn(dz, dz, __fmaf_rn(dy, dy, __fmul_rn(dx, dx)));
            }
            float h[32];
            window7<32>(d, h);
            float *hrow = hs + r * HP + 32 * warp;
#pragma unroll
            for (int q = 0; q < 32; ++q) hrow[q] = h[q];
        }
        __syncthreads();
        // ---- phase B: vertical sums for +o and -o, weights, accumulation -----------------
        if (t < TW) {
            const float geo = geo_l2_rt(i, j);
            float hv[TH + 6], D[TH];
            // +o: D_o(x, y) = sum_n H_o(x, y+n): H column t+3, rows 3 .. TH+8
#pragma unroll
            for (int q = 0; q < TH + 6; ++q) hv[q] = hs[(q + 3) * HP + t + 3];
            window7<TH>(hv, D);
#pragma unroll
            for (int r = 0; r < TH; ++r) {
                const float w = exp2f(__fmaf_rn(D[r], nl2, geo));
                const int pc = (r + 6 + i) * PW + t + 9 + j;
                ax[r] = __fmaf_rn(w, pr[pc], ax[r]);
                ay[r] = __fmaf_rn(w, pg[pc], ay[r]);
                az[r] = __fmaf_rn(w, pb[pc], az[r]);
                sw[r] = __fadd_rn(sw[r], w);
                cnt[r >> 2] += (w > wthr) ? (1u << (8 * (r & 3))) : 0u;
            }
            // -o: D_{-o}(x, y) = D_o(x-j, y-i): H column t+3-j, rows 3-i .. TH+8-i
#pragma unroll
            for (int q = 0; q < TH + 6; ++q) hv[q] = hs[(q + 3 - i) * HP + t + 3 - j];
            window7<TH>(hv, D);
#pragma unroll
            for (int r = 0; r < TH; ++r) {
                const float w = exp2f(__fmaf_rn(D[r], nl2, geo));
                const int pc = (r + 6 - i) * PW + t + 9 - j;
                ax[r] = __fmaf_rn(w, pr[pc], ax[r]);
                ay[r] = __fmaf_rn(w, pg[pc], ay[r]);
                az[r] = __fmaf_rn(w, pb[pc], az[r]);
                sw[r] = __fadd_rn(sw[r], w);
                cnt[r >> 2] += (w > wthr) ? (1u << (8 * (r & 3))) : 0u;
            }
        }
        __syncthreads();
    }
    const int x = x0 + t;
    if (t >= TW || x >= a.width) return;
    float4 *dst = (float4 *)a.dst;
#pragma unroll
    for (int r = 0; r < TH; ++r) {
        const int y = y0 + r;
        if (y >= a.row_end) break;
        const int pc = (r + 6) * PW + t + 9;
        const float4 c00 = make_float4(pr[pc], pg[pc], pb[pc], 0.0f);
        const int c = (int)((cnt[r >> 2] >> (8 * (r & 3))) & 0xffu);
        dst[(size_t)(y - a.dst_row_begin) * (size_t)a.width + x] = lerp_out(c00, ax[r], ay[r], az[r], sw[r], c, a);
    }
}
