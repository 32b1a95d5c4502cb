// nlm_box4.cu -- imageDenoising NLM filter (math per DESIGN.md reading
// R-O2), the separable box-sum form of nlm_box.cu with the input tile kept as ONE float4 plane
// (r, g, b, 1) instead of an (r, g) plane and a b plane:
//
//   D_o(x,y) = sum_{n,m=-3..3} d_o(x+m, y+n),   d_o(u,v) = |p(u+j, v+i) - p(u,v)|^2
//   H_o(u,v) = sum_m d_o(u+m, v)  (phase A),    D_o(x,y) = sum_n H_o(x, y+n)  (phase B),
//   D_{-o}(x,y) = D_o(x-j, y-i): one box sum serves the pair (o, -o)   -- as in nlm_box.cu.
//
// What the quad plane buys: a pixel is ONE 16-byte shared load (LDS.128) in both phases, and
// its (b, 1) half is a ready register pair, so the accumulation of (sum w b, sum w) is one
// FFMA2 with no pair-building move.  What it costs: 16 instead of 12 bytes per tile pixel, so
// two H buffers fit beside the plane instead of three -- 12 passes of G = 2 pairs (all
// packed: two window sums per FADD2) instead of 10 passes of 3 / 2 pairs.  The fourth
// component is set to 1 after staging (the input's alpha never enters the filter).
//
// CTA = 128 threads (4 warps); output tile TW = 122 columns x TH = 23 rows; shared memory:
// plane (TW+18) x (TH+12) float4 (odd pitch 141: LDS.128 of 8 lanes on 8 different rows or 8
// consecutive columns hit 8 different 16-byte bank groups) + 2 x 32 x 129 floats of H_o =
// 111 984 B -> 2 CTAs / SM.  Phase A: warp w = 32 H columns, lane = row (32 rows = TH + 9),
// sliding along the row over 38 difference values; phase B: thread = output column, all TH
// rows.  Two __syncthreads per pass.  Same arithmetic order per value as nlm_box.cu's packed
// offsets (every partial sum a sum of non-negative terms, <= 4 roundings deep).
#include "common.cuh"

namespace {

constexpr int TW = 122, TH = 23, NT = 128;
constexpr int AR = TH + 9;                  // phase-A rows (H rows): y0-6 .. y0+TH+3
constexpr int HC = TW + 6;                  // H columns: x0-3 .. x0+TW+3
constexpr int HP = HC + 1;                  // odd H pitch
constexpr int PC = TW + 18;                 // tile columns: x0-9 .. x0+TW+9
constexpr int PR = TH + 12;                 // tile rows:    y0-6 .. y0+TH+6
constexpr int PW = PC + 1;                  // odd plane pitch (float4 units)
constexpr int HBUF = AR * HP;               // floats per H buffer
constexpr int NPASS = 12;                   // 24 pairs, 2 per pass
static_assert(AR == 32 && HC == 4 * 32 && NT == 128, "phase A: one lane per row, one warp per 32 H columns");
static_assert(TW <= NT, "phase B: one thread per output column");

ORION_DEVICE float2 f2(float a, float b) { return make_float2(a, b); }
ORION_DEVICE float2 lo2(const float4 &v) { return make_float2(v.x, v.y); }
ORION_DEVICE float2 hi2(const float4 &v) { return make_float2(v.z, v.w); }

// |a - c|^2 = (dr^2 + dg^2) + db^2 with (r, g) on FADD2 / FMUL2 (R-NLM-FP), c negated once.
ORION_DEVICE float diff4(const float4 &a, float2 ncrg, float ncb)
{
    const float2 d = __fadd2_rn(lo2(a), ncrg);
    const float2 q = __fmul2_rn(d, d);
    const float db = __fadd_rn(a.z, ncb);
    return __fmaf_rn(db, db, __fadd_rn(q.x, q.y));
}

// Blocked 7-term window sums of two independent rows in lock step (fp32x2):
// out[k] = ((a[k]+a[k+1]) + (a[k+2]+a[k+3])) + ((a[k+4]+a[k+5]) + a[k+6]).
template <int N>
ORION_DEVICE void window7x2(const float2 (&a)[N + 6], float2 (&out)[N])
{
    float2 p[N + 5];
#pragma unroll
    for (int k = 0; k < N + 5; ++k) p[k] = __fadd2_rn(a[k], a[k + 1]);
#pragma unroll
    for (int k = 0; k < N; ++k) out[k] = __fadd2_rn(__fadd2_rn(p[k], p[k + 2]), __fadd2_rn(p[k + 4], a[k + 6]));
}

// Phase A for the offsets o1 = (i1, j1) and o2 = (i2, j2): lane = row, the warp's 32 H columns.
// SLIDE (i2 == i1, j2 == j1 + 1): the two shifted pixels of column q+1 include the second of
// column q, so a column costs two 16-byte loads (one shifted, the centre); otherwise three.
template <bool SLIDE>
ORION_DEVICE void phase_a(const float4 *pl, float *hs, int lane, int warp, int i1, int j1, int i2, int j2)
{
    const int rowc = lane * PW + 3 + 32 * warp;     // centre p(u, v), u = first difference column
    const int r1 = rowc + i1 * PW + j1;             // shifted p(u+j1, v+i1)
    const int r2 = rowc + i2 * PW + j2;             // shifted p(u+j2, v+i2)
    float4 s1 = pl[r1];
    float2 dp[38];
#pragma unroll
    for (int q = 0; q < 38; ++q) {
        float4 a1, a2;
        if (SLIDE) {
            a1 = s1;                                // p(u+q+j1)
            s1 = pl[r1 + q + 1];                    // p(u+q+j1+1) = p(u+q+j2)
            a2 = s1;
        } else {
            a1 = pl[r1 + q];
            a2 = pl[r2 + q];
        }
        const float4 c = pl[rowc + q];
        const float2 ncrg = f2(-c.x, -c.y);
        const float ncb = -c.z;
        dp[q] = f2(diff4(a1, ncrg, ncb), diff4(a2, ncrg, ncb));
    }
    float2 h[32];
    window7x2<32>(dp, h);
    float *h0 = hs + lane * HP + 32 * warp;
    float *h1 = h0 + HBUF;
#pragma unroll
    for (int q = 0; q < 32; ++q) {
        h0[q] = h[q].x;
        h1[q] = h[q].y;
    }
}

struct Acc {
    float2 axy[TH];               // (sum w*r, sum w*g)
    float2 azs[TH];               // (sum w*b, sum w)
    unsigned cnt[(TH + 3) / 4];   // 4 x 8-bit counts per word (<= 49)
};

ORION_DEVICE void count_above(Acc &A, int r, float w, float wthr)
{
    if (w > wthr) A.cnt[r >> 2] += 1u << (8 * (r & 3));
}

// Phase B for one pair (i, j) whose H_o lives in hb: thread t = output column x0+t.
ORION_DEVICE void phase_b(const float4 *pl, const float *hb, int t, int i, int j, float nl2, float wthr, Acc &A)
{
    const float geo = geo_l2_rt(i, j);
    float2 hv[TH + 6], D[TH];
#pragma unroll
    for (int q = 0; q < TH + 6; ++q) hv[q] = f2(hb[(q + 3) * HP + t + 3], hb[(q + 3 - i) * HP + t + 3 - j]);
    window7x2<TH>(hv, D);
    const float2 n2 = f2(nl2, nl2), g2 = f2(geo, geo);
#pragma unroll
    for (int r = 0; r < TH; ++r) {
        const float2 e = __ffma2_rn(D[r], n2, g2);
        const float wp = ex2(e.x), wm = ex2(e.y);
        const float4 pp = pl[(r + 6 + i) * PW + t + 9 + j];     // p(x+j, y+i)
        const float4 pm = pl[(r + 6 - i) * PW + t + 9 - j];     // p(x-j, y-i)
        A.axy[r] = __ffma2_rn(f2(wp, wp), lo2(pp), A.axy[r]);
        A.azs[r] = __ffma2_rn(f2(wp, wp), hi2(pp), A.azs[r]);
        A.axy[r] = __ffma2_rn(f2(wm, wm), lo2(pm), A.axy[r]);
        A.azs[r] = __ffma2_rn(f2(wm, wm), hi2(pm), A.azs[r]);
        count_above(A, r, wp, wthr);
        count_above(A, r, wm, wthr);
    }
}

// Passes (i1, j1, i2, j2): the 24 half-plane offsets (i = 0: j = 1..3; i = 1..3: j = -3..3)
// exactly once.  Ten passes of two consecutive column offsets on one row (sliding loads), and
// the four j = 3 offsets left over paired across rows in two general passes.
__constant__ int kPass[NPASS][4] = {
    {0, 1, 0, 2},
    {1, -3, 1, -2}, {1, -1, 1, 0}, {1, 1, 1, 2},
    {2, -3, 2, -2}, {2, -1, 2, 0}, {2, 1, 2, 2},
    {3, -3, 3, -2}, {3, -1, 3, 0}, {3, 1, 3, 2},
    {0, 3, 1, 3}, {2, 3, 3, 3}};
constexpr int NSLIDE = 10;

__device__ __forceinline__ void nlm_box4_body(const orion_kargs &a)
{
    extern __shared__ float4 smem4[];
    float4 *pl = smem4;                                          // (r, g, b, 1) plane
    float *hs = reinterpret_cast<float *>(pl + PR * PW);         // 2 buffers of H_o: AR rows x HP

    const int tid = threadIdx.x;
    const int lane = tid & 31, warp = tid >> 5;
    const int x0 = blockIdx.x * TW;
    const int y0 = a.row_begin + blockIdx.y * TH;
    {   // stage the tile (clamp-to-edge in global coords): one 16-byte cp.async per pixel, all of
        // the thread's copies in flight at once; then the fourth component := 1 (own pixels)
        const float4 *src = (const float4 *)a.src;
#pragma unroll 4
        for (int idx = tid; idx < PC * PR; idx += NT) {
            const int ty = idx / PC, tx = idx - ty * PC;
            const int gx = clampi(x0 - 9 + tx, 0, a.width - 1);
            const int gy = slab_row(a, y0 - 6 + ty);
            cpa16(pl + ty * PW + tx, src + (size_t)(gy - a.src_row_begin) * (size_t)a.width + gx);
        }
        cp_async_wait_all();
#pragma unroll 4
        for (int idx = tid; idx < PC * PR; idx += NT) {
            const int ty = idx / PC, tx = idx - ty * PC;
            reinterpret_cast<float *>(pl + ty * PW + tx)[3] = 1.0f;
        }
    }
    __syncthreads();

    const float nl2 = a.fparam[0];
    const float wthr = a.fparam[2];
    const int t = tid;
    Acc A;
    {
        const unsigned c1 = (1.0f > wthr) ? 1u : 0u;   // centre offset: D = 0, w = 1 exactly
#pragma unroll
        for (int r = 0; r < TH; ++r) {
            const float4 pc = pl[(r + 6) * PW + t + 9];
            A.axy[r] = lo2(pc);
            A.azs[r] = f2(pc.z, 1.0f);
        }
#pragma unroll
        for (int q = 0; q < (TH + 3) / 4; ++q) A.cnt[q] = c1 * 0x01010101u;
    }

#pragma unroll 1
    for (int ps = 0; ps < NPASS; ++ps) {
        const int i1 = kPass[ps][0], j1 = kPass[ps][1], i2 = kPass[ps][2], j2 = kPass[ps][3];
        if (ps < NSLIDE)
            phase_a<true>(pl, hs, lane, warp, i1, j1, i2, j2);
        else
            phase_a<false>(pl, hs, lane, warp, i1, j1, i2, j2);
        __syncthreads();
        if (t < TW) {
            phase_b(pl, hs, t, i1, j1, nl2, wthr, A);
            phase_b(pl, hs + HBUF, t, i2, j2, nl2, wthr, A);
        }
        __syncthreads();
    }
    const int x = x0 + t;
    if (t >= TW || x >= a.width) return;
#pragma unroll
    for (int r = 0; r < TH; ++r) {
        const int y = y0 + r;
        if (y >= a.row_end) break;
        const float4 pc = pl[(r + 6) * PW + t + 9];
        const float4 c00 = make_float4(pc.x, pc.y, pc.z, 0.0f);
        const int c = (int)((A.cnt[r >> 2] >> (8 * (r & 3))) & 0xffu);
        store_out(a, x, y, lerp_out(c00, A.axy[r].x, A.axy[r].y, A.azs[r].x, A.azs[r].y, c, a));
    }
    fanout_column(a, x, y0, min(y0 + TH, a.row_end));
}

}  // namespace

// Two pairs per pass over a (r, g, b, 1) float4 plane: 78 960 + 2 x 16 512 = 111 984 B of shared memory.
extern "C" __global__ void __launch_bounds__(128) orion_nlm_box4_f4_128(orion_kargs a) { ORION_PROBE(a); nlm_box4_body(a); }
