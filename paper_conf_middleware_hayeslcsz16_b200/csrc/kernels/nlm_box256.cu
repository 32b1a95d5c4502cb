// nlm_box256.cu -- the NLM box-sum kernel of nlm_box.cu (same identities: separable box
// sums, symmetric offset pairs, up to 3 pairs per pass sharing a sliding shifted window,
// fixed-point exact integer windows) with TWICE the warps per tile: 256 threads, so the SM
// holds 16 warps instead of 8 at the same shared-memory footprint (2 CTAs/SM) and the
// sliding-window dependency chains of one warp are hidden behind the others.
//
//   phase A: warp w (0..7) computes H_o for H columns [16w, 16w+16) of every offset of the
//            pass; lane = row (32 rows = TH + 9); 22 differences per lane and offset.
//   phase B: thread (t, h): output column x0+t, rows 0..11 (h = 0) or 11..22 (h = 1; row 11
//            is computed by both halves and written by h = 0); vertical windows of 12.
// Results equal nlm_box.cu's integer kernel bit for bit (same quantisation, exact sums, same
// accumulation order per pixel).
#include "common.cuh"

namespace {

constexpr int TW = 122, TH = 23, NT = 256;
constexpr int AR = TH + 9;                  // H rows: y0-6 .. y0+TH+3
constexpr int HC = TW + 6;                  // H columns: x0-3 .. x0+TW+3
constexpr int HP = HC + 1;                  // odd H pitch
constexpr int PC = TW + 18;                 // image tile columns: x0-9 .. x0+TW+9
constexpr int PR = TH + 12;                 // image tile rows:    y0-6 .. y0+TH+6
constexpr int PW = PC + 1;                  // odd plane pitch
constexpr int HBUF = AR * HP;
constexpr int SEG = 16;                     // H columns per warp in phase A
constexpr int RH = 12;                      // rows per phase-B thread
static_assert(AR == 32 && HC == 8 * SEG, "phase A: one lane per row, 8 warps x 16 H columns");

constexpr float kQScale = 2097152.0f;            // 2^21
constexpr float kQMagic = 8388608.0f;            // 2^23
constexpr unsigned kQMagicBits = 0x4B000000u;    // bits of 2^23

ORION_DEVICE unsigned quant(float d) { return __float_as_uint(__fmaf_rn(d, kQScale, kQMagic)); }

ORION_DEVICE float diff2(float ar, float ag, float ab, float br, float bg, float bb)
{
    const float dx = __fsub_rn(ar, br), dy = __fsub_rn(ag, bg), dz = __fsub_rn(ab, bb);
    return __fmaf_rn(dz, dz, __fmaf_rn(dy, dy, __fmul_rn(dx, dx)));
}

ORION_DEVICE float2 fma2(float2 a, float2 b, float2 c) { return __ffma2_rn(a, b, c); }

template <int G>
ORION_DEVICE void phase_a(const float *pr, const float *pg, const float *pb, unsigned *hs, int lane, int warp, int i,
                          int j1)
{
    const int cb = 3 + SEG * warp;
    const int rowc = lane * PW + cb;
    const int rows = rowc + i * PW + j1;
    float wr[G], wg[G], wb[G];
#pragma unroll
    for (int g = 0; g < G - 1; ++g) {
        wr[g + 1] = pr[rows + g];
        wg[g + 1] = pg[rows + g];
        wb[g + 1] = pb[rows + g];
    }
    unsigned q[G][SEG + 6];
#pragma unroll
    for (int c = 0; c < SEG + 6; ++c) {
#pragma unroll
        for (int g = 0; g < G - 1; ++g) {
            wr[g] = wr[g + 1];
            wg[g] = wg[g + 1];
            wb[g] = wb[g + 1];
        }
        wr[G - 1] = pr[rows + c + G - 1];
        wg[G - 1] = pg[rows + c + G - 1];
        wb[G - 1] = pb[rows + c + G - 1];
        const float cr = pr[rowc + c], cg = pg[rowc + c], cbv = pb[rowc + c];
#pragma unroll
        for (int g = 0; g < G; ++g) q[g][c] = quant(diff2(wr[g], wg[g], wb[g], cr, cg, cbv));
    }
#pragma unroll
    for (int g = 0; g < G; ++g) {
        unsigned s = q[g][0] + q[g][1] + q[g][2] + q[g][3] + q[g][4] + q[g][5] + q[g][6] - 7u * kQMagicBits;
        unsigned *hrow = hs + g * HBUF + lane * HP + SEG * warp;
        hrow[0] = s;
#pragma unroll
        for (int k = 1; k < SEG; ++k) {
            s = s + q[g][k + 6] - q[g][k - 1];
            hrow[k] = s;
        }
    }
}

struct Acc {
    float2 axy[RH];               // (sum w*r, sum w*g)
    float2 azs[RH];               // (sum w*b, sum w)
    unsigned cnt[RH / 4];         // 4 x 8-bit counts per word (<= 49)
};

// Phase B for one pair (i, j): column t, tile rows r0 .. r0+RH-1.
ORION_DEVICE void phase_b(const float *pr, const float *pg, const float *pb, const unsigned *hb, int t, int r0, int i,
                          int j, float nl2q, float wthr, Acc &A)
{
    const float geo = geo_l2_rt(i, j);
    unsigned sp = 0, sm = 0;
    unsigned hp[RH + 6], hm[RH + 6];
#pragma unroll
    for (int c = 0; c < RH + 6; ++c) {
        hp[c] = hb[(r0 + c + 3) * HP + t + 3];           // +o: H column t+3
        hm[c] = hb[(r0 + c + 3 - i) * HP + t + 3 - j];   // -o: H column t+3-j, shifted by -i rows
    }
#pragma unroll
    for (int r = 0; r < RH; ++r) {
        if (r == 0) {
            sp = hp[0] + hp[1] + hp[2] + hp[3] + hp[4] + hp[5] + hp[6];
            sm = hm[0] + hm[1] + hm[2] + hm[3] + hm[4] + hm[5] + hm[6];
        } else {
            sp = sp + hp[r + 6] - hp[r - 1];
            sm = sm + hm[r + 6] - hm[r - 1];
        }
        const float wp = ex2(__fmaf_rn(__uint2float_rn(sp), nl2q, geo));
        const float wm = ex2(__fmaf_rn(__uint2float_rn(sm), nl2q, geo));
        const int pp = (r0 + r + 6 + i) * PW + t + 9 + j;      // p(x+j, y+i)
        const int pm = (r0 + r + 6 - i) * PW + t + 9 - j;      // p(x-j, y-i)
        A.axy[r] = fma2(make_float2(wp, wp), make_float2(pr[pp], pg[pp]), A.axy[r]);
        A.azs[r] = fma2(make_float2(wp, wp), make_float2(pb[pp], 1.0f), A.azs[r]);
        A.axy[r] = fma2(make_float2(wm, wm), make_float2(pr[pm], pg[pm]), A.axy[r]);
        A.azs[r] = fma2(make_float2(wm, wm), make_float2(pb[pm], 1.0f), A.azs[r]);
        A.cnt[r >> 2] += (((wp > wthr) ? 1u : 0u) + ((wm > wthr) ? 1u : 0u)) << (8 * (r & 3));
    }
}

__constant__ int kPass3[10][3] = {
    {0, 1, 3}, {1, -3, 3}, {1, 0, 2}, {1, 2, 2}, {2, -3, 3}, {2, 0, 2}, {2, 2, 2}, {3, -3, 3}, {3, 0, 2}, {3, 2, 2}};

}  // namespace

// 3 planar planes + 3 H buffers = 108 756 B of shared memory; 2 CTAs x 8 warps per SM.
extern "C" __global__ void __launch_bounds__(256) orion_nlm_box256_f4_256(orion_kargs a)
{
    ORION_PROBE(a);
    extern __shared__ float4 smem4[];
    float *pr = reinterpret_cast<float *>(smem4);
    float *pg = pr + PR * PW;
    float *pb = pg + PR * PW;
    unsigned *hs = reinterpret_cast<unsigned *>(pb + PR * PW);

    const int tid = threadIdx.x;
    const int lane = tid & 31, warp = tid >> 5;
    const int x0 = blockIdx.x * TW;
    const int y0 = a.row_begin + blockIdx.y * TH;
    {
        const float4 *src = (const float4 *)a.src;
#pragma unroll 4
        for (int idx = tid; idx < PC * PR; idx += NT) {
            const int ty = idx / PC, tx = idx - ty * PC;
            const int gx = clampi(x0 - 9 + tx, 0, a.width - 1);
            const int gy = slab_row(a, y0 - 6 + ty);
            const float *g = (const float *)(src + (size_t)(gy - a.src_row_begin) * (size_t)a.width + gx);
            cpa4(pr + ty * PW + tx, g);        // cp.async: all copies in flight at once
            cpa4(pg + ty * PW + tx, g + 1);
            cpa4(pb + ty * PW + tx, g + 2);
        }
        cp_async_wait_all();
    }
    __syncthreads();

    const float nl2q = a.fparam[0] * (1.0f / kQScale);
    const float wthr = a.fparam[2];
    const int t = tid & 127, h = tid >> 7;
    const int r0 = h ? TH - RH : 0;              // rows 0..11 or 11..22
    Acc A;
    {
        const unsigned c1 = (1.0f > wthr) ? 1u : 0u;   // centre offset: D = 0, w = 1 exactly
#pragma unroll
        for (int r = 0; r < RH; ++r) {
            const int pc = (r0 + r + 6) * PW + t + 9;
            A.axy[r] = make_float2(pr[pc], pg[pc]);
            A.azs[r] = make_float2(pb[pc], 1.0f);
        }
#pragma unroll
        for (int q = 0; q < RH / 4; ++q) A.cnt[q] = c1 * 0x01010101u;
    }

#pragma unroll 1
    for (int ps = 0; ps < 10; ++ps) {
        const int i = kPass3[ps][0], j1 = kPass3[ps][1], G = kPass3[ps][2];
        if (G == 3)
            phase_a<3>(pr, pg, pb, hs, lane, warp, i, j1);
        else
            phase_a<2>(pr, pg, pb, hs, lane, warp, i, j1);
        __syncthreads();
        if (t < TW) {
#pragma unroll 1
            for (int g = 0; g < G; ++g) phase_b(pr, pg, pb, hs + g * HBUF, t, r0, i, j1 + g, nl2q, wthr, A);
        }
        __syncthreads();
    }
    const int x = x0 + t;
    if (t >= TW || x >= a.width) return;
#pragma unroll
    for (int r = 0; r < RH; ++r) {
        if (h && r == 0) continue;               // row 11 belongs to the upper half
        const int y = y0 + r0 + r;
        if (y >= a.row_end) break;
        const int pc = (r0 + r + 6) * PW + t + 9;
        const float4 c00 = make_float4(pr[pc], pg[pc], pb[pc], 0.0f);
        const int c = (int)((A.cnt[r >> 2] >> (8 * (r & 3))) & 0xffu);
        store_out(a, x, y, lerp_out(c00, A.axy[r].x, A.axy[r].y, A.azs[r].x, A.azs[r].y, c, a));
    }
    fanout_column(a, x, y0 + r0 + (h ? 1 : 0), min(y0 + r0 + RH, a.row_end));
}
