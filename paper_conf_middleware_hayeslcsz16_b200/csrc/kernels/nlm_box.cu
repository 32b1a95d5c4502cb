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
// (3) Pairs sharing the row offset i and consecutive column offsets j = j1 .. j1+G-1
//     are processed in one pass: along a phase-A row the shifted pixels p(u+j, v+i) of
//     the G offsets form a sliding window, so each new column costs one shifted load for
//     all G differences (and one centre load), instead of G of each.
// All three are exact identities; only the order of the fp32 additions differs from the
// definition (every partial sum is a sum of non-negative terms, at most 4 roundings
// deep: DESIGN.md §7 gives the error budget against the 1e-5 tolerance).
//
// CTA = 128 threads (4 warps); output tile TW = 122 columns x TH = 23 rows.
// Shared memory: the input tile (TW+18) x (TH+12) with a 9-column / 6-row
// clamp-to-edge halo as an (r, g) float2 plane and a b plane (odd pitch; one LDS.64 + one
// LDS per pixel, conflict-free for both access patterns below), and three buffers of
// H_o, 32 rows x 128 columns each (odd pitch).  Per pass:
//   phase A: warp w computes H_o for columns [32w, 32w+32) of each buffer; lane = row
//            (32 rows = TH + 9), sliding along the row over 38 difference values per
//            offset.  Lanes touch 32 different rows of odd-pitch arrays: conflict-free.
//   phase B: thread t owns output column x0+t and all TH rows: vertical 7-sums of
//            H_o down column t+3 give D_o(x, .), and down column t+3-j, shifted by -i
//            rows, give D_{-o}(x, .); weights w = 2^(D * (-Noise log2 e) + geo) and
//            the accumulation of w*p, w and [w > wthr] for both offsets.  Lanes touch
//            consecutive columns: conflict-free.
// Two __syncthreads per pass; eight passes of three pairs, 108.8 KB of shared memory (2 CTAs/SM).
// (Round 1 measured and removed: one pair per pass in 24 passes at 3 CTAs/SM, 0.295 ms at C2;
// exact fixed-point integer windows, 0.27 ms; a 256-thread CTA, 0.28 ms; a (r, g, b, 1)
// float4 tile plane with two pairs per pass, 0.272 ms -- against 0.234 ms for this form.)
#include "common.cuh"

#define PB_R 3   // window radius
#define PB_B 3   // patch radius

namespace {

// NLMB_WIDE (nlm_boxw.cu): TW = 128 output columns, every phase-B thread busy, phase-A warps of
// 34 H columns (136 >= TW + 6), the tile two columns wider on the right; 115 188 B of shared
// memory, still 2 CTAs/SM.  A 2048-wide frame is then 16 tile columns instead of 17.
#ifdef NLMB_WIDE
constexpr int TW = 128, HWARP = 34;
#else
constexpr int TW = 122, HWARP = 32;
#endif
constexpr int TH = 23, NT = 128;
constexpr int ND = HWARP + 6;               // differences a phase-A lane slides over
constexpr int AR = TH + 9;                  // phase-A rows (H rows): y0-6 .. y0+TH+3
constexpr int HC = 4 * HWARP;               // H columns: x0-3 .. (>= x0+TW+3)
constexpr int HP = HC + 1;                  // odd H pitch
constexpr int PC = HC + 12;                 // image tile columns: x0-9 .. (>= x0+TW+9)
constexpr int PR = TH + 12;                 // image tile rows:    y0-6 .. y0+TH+6
constexpr int PW = PC + 1;                  // odd plane pitch
constexpr int HBUF = AR * HP;               // floats per H buffer
static_assert(AR == 32 && HC >= TW + 6 && NT == 128, "phase A: one lane per row, 4 warps of HWARP H columns");
static_assert(TW <= NT, "phase B: one thread per output column");

// Packed fp32x2 arithmetic (sm_100 FADD2 / FMUL2 / FFMA2): two independent IEEE
// round-to-nearest operations per instruction, bit-identical to the scalar .rn forms.
ORION_DEVICE float2 sub2(float2 a, float2 b) { return __fadd2_rn(a, make_float2(-b.x, -b.y)); }
ORION_DEVICE float2 mul2(float2 a, float2 b) { return __fmul2_rn(a, b); }
ORION_DEVICE float2 fma2(float2 a, float2 b, float2 c) { return __ffma2_rn(a, b, c); }
ORION_DEVICE float add1(float a, float b) { return __fadd_rn(a, b); }
ORION_DEVICE float2 add1(float2 a, float2 b) { return __fadd2_rn(a, b); }

// Blocked 7-term window sums of a[0 .. N+5]: out[k] = a[k] + ... + a[k+6] evaluated as
// ((a[k]+a[k+1]) + (a[k+2]+a[k+3])) + ((a[k+4]+a[k+5]) + a[k+6]) -- 4 additions per
// output with the pair sums shared; every partial sum is a sum of non-negatives.
// T = float, or float2 for two independent windows in lock step.
template <int N, typename T>
ORION_DEVICE void window7(const T (&a)[N + 6], T (&out)[N])
{
    T p[N + 5];
#pragma unroll
    for (int k = 0; k < N + 5; ++k) p[k] = add1(a[k], a[k + 1]);
#pragma unroll
    for (int k = 0; k < N; ++k) out[k] = add1(add1(p[k], p[k + 2]), add1(p[k + 4], a[k + 6]));
}

// |a - c|^2 with the (r, g) channels packed: a.rg + (-c.rg) on FADD2, squares on FMUL2, then
// (dr^2 + dg^2) + db^2.  A sum of non-negative terms, 3 roundings deep.
ORION_DEVICE float2 neg2(float2 a) { return make_float2(-a.x, -a.y); }
ORION_DEVICE float diff2rg(float2 arg, float ab, float2 ncrg, float cb)
{
    const float2 d = __fadd2_rn(arg, ncrg);
    const float2 q = __fmul2_rn(d, d);
    const float db = __fsub_rn(ab, cb);
    return __fmaf_rn(db, db, __fadd_rn(q.x, q.y));
}

// Phase A for G offsets (i, j1 .. j1+G-1): lane = row r, warp's 32 H columns.  Differences
// are channel-packed (diff2rg); the window sums of offsets g = 0, 1 run packed (fp32x2),
// offset g = 2 scalar.
// VERT: the G offsets (i .. i+G-1, j1) -- one column offset on G rows -- with G shifted loads per
// column instead of one (the j = 3 offsets of rows 1..3 in one pass instead of three).
template <int G, bool VERT = false>
ORION_DEVICE void phase_a(const float2 *prg, const float *pb, float *hs, int lane, int warp, int i,
                          int j1)
{
    const int cb = 3 + HWARP * warp;            // tile column of u for the first difference
    const int rowc = lane * PW + cb;            // centre p(u, v)
    const int rows = rowc + i * PW + j1;        // shifted p(u+j1, v+i)
    // the shifted window holds columns q + j1 .. q + j1 + G - 1 at step q
    float2 wrg[G];
    float wb[G];
#pragma unroll
    for (int g = 0; g < G - 1; ++g) {
        if (VERT) break;
        wrg[g + 1] = prg[rows + g];
        wb[g + 1] = pb[rows + g];
    }
    constexpr int GP = G / 2;                   // packed offset pairs (0 or 1)
    constexpr int GS = G - 2 * GP;              // scalar offsets left (0 or 1)
    float2 dp[GP > 0 ? ND : 1];
    float ds[GS > 0 ? ND : 1];
#pragma unroll
    for (int q = 0; q < ND; ++q) {
        if (VERT) {
#pragma unroll
            for (int g = 0; g < G; ++g) {
                wrg[g] = prg[rows + g * PW + q];
                wb[g] = pb[rows + g * PW + q];
            }
        } else {
#pragma unroll
            for (int g = 0; g < G - 1; ++g) {
                wrg[g] = wrg[g + 1];
                wb[g] = wb[g + 1];
            }
            wrg[G - 1] = prg[rows + q + G - 1];
            wb[G - 1] = pb[rows + q + G - 1];
        }
        const float2 ncrg = neg2(prg[rowc + q]);
        const float cbv = pb[rowc + q];
        if (GP > 0)
            dp[GP > 0 ? q : 0] = make_float2(diff2rg(wrg[0], wb[0], ncrg, cbv),
                                             diff2rg(wrg[GP > 0 ? 1 : 0], wb[GP > 0 ? 1 : 0], ncrg, cbv));
        if (GS > 0) ds[GS > 0 ? q : 0] = diff2rg(wrg[G - 1], wb[G - 1], ncrg, cbv);
    }
    if (GP > 0) {
        float2 h[HWARP];
        window7<HWARP>(*reinterpret_cast<float2(*)[ND]>(&dp), h);
        float *h0 = hs + lane * HP + HWARP * warp;
        float *h1 = h0 + HBUF;
#pragma unroll
        for (int q = 0; q < HWARP; ++q) {
            h0[q] = h[q].x;
            h1[q] = h[q].y;
        }
    }
    if (GS > 0) {
        float h[HWARP];
        window7<HWARP>(*reinterpret_cast<float(*)[ND]>(&ds), h);
        float *h2 = hs + (G - 1) * HBUF + lane * HP + HWARP * warp;
#pragma unroll
        for (int q = 0; q < HWARP; ++q) h2[q] = h[q];
    }
}

struct Acc {
    float2 axy[TH];               // (sum w*r, sum w*g)
    float2 azs[TH];               // (sum w*b, sum w)
    unsigned cnt[(TH + 3) / 4];   // 4 x 8-bit counts per word (<= 49)
};

// [w > wthr] into row r's 8-bit count: FSETP + one predicated IADD of an immediate.  Decided on
// the exponent: w = 2^e > wthr <=> e > log2(wthr) (ethr, host-computed), so the compare does not
// wait for MUFU.EX2; the two tests differ only within ex2.approx's 2 ulp of the threshold, inside
// the ambiguous-weight band (reading R-AMB).
ORION_DEVICE void count_above(Acc &A, int r, float e, float ethr)
{
    if (e > ethr) A.cnt[r >> 2] += 1u << (8 * (r & 3));
}

// Phase B for one pair (i, j) whose H_o lives in hb: thread t = output column x0+t.  The
// +o and -o vertical windows run packed (fp32x2), as do their exponent arguments and the
// (r, g) / (b, weight) accumulations.
ORION_DEVICE void phase_b(const float2 *prg, const float *pb, const float *hb, int t, int i, int j,
                          float nl2, float ethr, Acc &A)
{
    const float geo = geo_l2_rt(i, j);
    // x: D_o(x, y) = sum_n H_o(x, y+n) -- H column t+3, rows 3 .. TH+8
    // y: D_{-o}(x, y) = D_o(x-j, y-i)  -- H column t+3-j, rows 3-i .. TH+8-i
    float2 hv[TH + 6], D[TH];
#pragma unroll
    for (int q = 0; q < TH + 6; ++q) hv[q] = make_float2(hb[(q + 3) * HP + t + 3], hb[(q + 3 - i) * HP + t + 3 - j]);
    window7<TH>(hv, D);
    const float2 n2 = make_float2(nl2, nl2), g2 = make_float2(geo, geo);
#pragma unroll
    for (int r = 0; r < TH; ++r) {
        const float2 e = fma2(D[r], n2, g2);
        const float wp = ex2(e.x), wm = ex2(e.y);
        const int pp = (r + 6 + i) * PW + t + 9 + j;      // p(x+j, y+i)
        const int pm = (r + 6 - i) * PW + t + 9 - j;      // p(x-j, y-i)
        A.axy[r] = fma2(make_float2(wp, wp), prg[pp], A.axy[r]);
        A.azs[r] = fma2(make_float2(wp, wp), make_float2(pb[pp], 1.0f), A.azs[r]);
        A.axy[r] = fma2(make_float2(wm, wm), prg[pm], A.axy[r]);
        A.azs[r] = fma2(make_float2(wm, wm), make_float2(pb[pm], 1.0f), A.azs[r]);
        count_above(A, r, e.x, ethr);
        count_above(A, r, e.y, ethr);
    }
}

// The 24 half-plane pairs in eight passes of three offsets, (i, j1, vert): seven sliding passes
// (i, j1 .. j1+2) and one vertical pass (1 .. 3, 3) -- every pair exactly once.
__constant__ int kPass8[8][3] = {
    {0, 1, 0}, {1, -3, 0}, {1, 0, 0}, {2, -3, 0}, {2, 0, 0}, {3, -3, 0}, {3, 0, 0}, {1, 3, 1}};

__device__ __forceinline__ void nlm_box_body(const orion_kargs &a)
{
    extern __shared__ float4 smem4[];
    float2 *prg = reinterpret_cast<float2 *>(smem4);             // (r, g) plane
    float *pb = reinterpret_cast<float *>(prg + PR * PW);         // b plane
    float *hs = pb + PR * PW;               // 3 buffers of H_o: AR rows x HP

    const int tid = threadIdx.x;
    const int lane = tid & 31, warp = tid >> 5;
    const int x0 = blockIdx.x * TW;
    const int y0 = a.row_begin + blockIdx.y * TH;
    {   // stage the planar tile (clamp-to-edge in global coords): per pixel one 8-byte (r, g)
        // and one 4-byte b cp.async, all of the thread's copies in flight at once
        const float4 *src = (const float4 *)a.src + frame_px(a);
#pragma unroll 4
        for (int idx = tid; idx < PC * PR; idx += NT) {
            const int ty = idx / PC, tx = idx - ty * PC;
            const int gx = clampi(x0 - 9 + tx, 0, a.width - 1);
            const int gy = slab_row(a, y0 - 6 + ty);
            const float *g = (const float *)(src + (size_t)(gy - a.src_row_begin) * (size_t)a.width + gx);
            cpa8(prg + ty * PW + tx, g);
            cpa4(pb + ty * PW + tx, g + 2);
        }
        cp_async_wait_all();
    }
    __syncthreads();

    const float nl2 = a.fparam[0];
    const float wthr = a.fparam[2];
    const float ethr = a.fparam[3];          // log2(wthr)
    const int t = tid;
    Acc A;
    {
        const unsigned c1 = (1.0f > wthr) ? 1u : 0u;   // centre offset: D = 0, w = 1 exactly
#pragma unroll
        for (int r = 0; r < TH; ++r) {
            const int pc = (r + 6) * PW + t + 9;
            A.axy[r] = prg[pc];
            A.azs[r] = make_float2(pb[pc], 1.0f);
        }
#pragma unroll
        for (int q = 0; q < (TH + 3) / 4; ++q) A.cnt[q] = c1 * 0x01010101u;
    }

#pragma unroll 1
    for (int ps = 0; ps < 8; ++ps) {
        const int i = kPass8[ps][0], j1 = kPass8[ps][1], vert = kPass8[ps][2];
        if (vert)
            phase_a<3, true>(prg, pb, hs, lane, warp, i, j1);
        else
            phase_a<3>(prg, pb, hs, lane, warp, i, j1);
        __syncthreads();
        if (t < TW) {
#pragma unroll 1
            for (int g = 0; g < 3; ++g) {
                const int ig = vert ? i + g : i, jg = vert ? j1 : j1 + g;
                phase_b(prg, pb, hs + g * HBUF, t, ig, jg, nl2, ethr, A);
            }
        }
        __syncthreads();
    }
    const int x = x0 + t;
    if (t >= TW || x >= a.width) return;
#pragma unroll
    for (int r = 0; r < TH; ++r) {
        const int y = y0 + r;
        if (y >= a.row_end) break;
        const int pc = (r + 6) * PW + t + 9;
        const float4 c00 = make_float4(prg[pc].x, prg[pc].y, pb[pc], 0.0f);
        const int c = (int)((A.cnt[r >> 2] >> (8 * (r & 3))) & 0xffu);
        store_out(a, x, y, lerp_out(c00, A.axy[r].x, A.axy[r].y, A.azs[r].x, A.azs[r].y, c, a));
    }
    fanout_column(a, x, y0, min(y0 + TH, a.row_end));
}

}  // namespace

#ifndef NLMB_WIDE
// 122-column tiles, three pairs per pass: 3 planar planes + 3 H buffers = 108 756 B of shared memory.
extern "C" __global__ void __launch_bounds__(128) orion_nlm_box3_f4_128(orion_kargs a) { ORION_PROBE(a); nlm_box_body(a); }
#else
// 128-column tiles, three pairs per pass: 115 188 B of shared memory.
extern "C" __global__ void __launch_bounds__(128) orion_nlm_boxw3_f4_128(orion_kargs a) { ORION_PROBE(a); nlm_box_body(a); }
#endif
