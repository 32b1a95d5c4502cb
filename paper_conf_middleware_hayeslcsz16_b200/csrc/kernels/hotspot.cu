// hotspot.cu -- Rodinia-style 2-D thermal stencil, one explicit step per launch
// (Table 2, Rodinia [6] P:L1147; update rule per DESIGN.md reading
// R-O3, constants per reading R-A15):
//   T' = T + sdc * ( P + (S + N - 2T)*ry + (E + W - 2T)*rx + (amb - T)*rz )
// with clamp-to-edge neighbours, evaluated in fp32 in exactly this order, one rounding per
// operation with the products that feed a sum fused (reading R-HS-FP; 9 operations):
//   a = fma(T,-2,S+N); b = fma(T,-2,E+W); d = amb-T; acc = fma(rz,d,fma(rx,b,fma(ry,a,P)));
//   T' = fma(sdc, acc, T)
//
// HBM-bound: 12 algorithmic bytes per cell-step (read T and P, write T').  Each warp
// owns 128 consecutive columns (4 per lane, 16-byte vector loads and stores) and walks
// a strip of RY rows top to bottom keeping N / T / S in registers, so every row of T is
// read from DRAM once per strip; W and E of the lane's 4 cells come from the
// neighbouring lanes by shuffle, lanes 0/31 fetch their outer neighbour (an L1/L2 hit:
// the neighbouring warp reads that line).  Grids whose width is not a multiple of 4
// (rows not 16-byte aligned) take a scalar path with the same arithmetic.
#include "common.cuh"

ORION_DEVICE float hs_cell(float T, float N, float S, float E, float Wv, float P, const float (&c)[5])
{
    const float av = __fmaf_rn(T, -2.0f, __fadd_rn(S, N));
    const float bv = __fmaf_rn(T, -2.0f, __fadd_rn(E, Wv));
    const float dv = __fsub_rn(c[4], T);
    const float acc = __fmaf_rn(c[3], dv, __fmaf_rn(c[1], bv, __fmaf_rn(c[2], av, P)));
    return __fmaf_rn(c[0], acc, T);
}

// The same update for a lane's 4 consecutive cells (a float4 of one row) on the packed fp32x2
// pipe (FADD2 / FFMA2: two independent IEEE .rn operations per instruction, bit-identical to
// hs_cell): cells (x, y) and (z, w) run as two pairs.  E + W of a pair is not a register pair
// of the row (cell x needs T.y + Wv, cell y T.z + T.x), so those two sums are scalar FADDs
// written straight into a pair; everything else is 8 packed instructions per 2 cells instead
// of 18 scalar ones.  Ev / Wv: east neighbour of cell w, west neighbour of cell x.
ORION_DEVICE float2 hs_pair(float2 T, float2 N, float2 S, float2 ew, float2 P, const float (&c)[5])
{
    const float2 av = __ffma2_rn(T, make_float2(-2.0f, -2.0f), __fadd2_rn(S, N));
    const float2 bv = __ffma2_rn(T, make_float2(-2.0f, -2.0f), ew);
    const float2 dv = __fadd2_rn(make_float2(c[4], c[4]), make_float2(-T.x, -T.y));
    const float2 acc = __ffma2_rn(make_float2(c[3], c[3]), dv,
                                  __ffma2_rn(make_float2(c[1], c[1]), bv,
                                             __ffma2_rn(make_float2(c[2], c[2]), av, P)));
    return __ffma2_rn(make_float2(c[0], c[0]), acc, T);
}
ORION_DEVICE float4 hs_cell4(float4 T, float4 N, float4 S, float Ev, float Wv, float4 P, const float (&c)[5])
{
    const float2 lo = hs_pair(make_float2(T.x, T.y), make_float2(N.x, N.y), make_float2(S.x, S.y),
                              make_float2(__fadd_rn(T.y, Wv), __fadd_rn(T.z, T.x)), make_float2(P.x, P.y), c);
    const float2 hi = hs_pair(make_float2(T.z, T.w), make_float2(N.z, N.w), make_float2(S.z, S.w),
                              make_float2(__fadd_rn(T.w, T.y), __fadd_rn(Ev, T.z)), make_float2(P.z, P.w), c);
    return make_float4(lo.x, lo.y, hi.x, hi.y);
}

template <int BY, int RY>
__device__ __forceinline__ void hotspot_body(const orion_kargs &a)
{
    const float *tin = (const float *)a.src;
    const float *pw = (const float *)a.aux;
    float *tout = (float *)a.dst;
    const int W = a.width, H = a.height;
    const int lane = threadIdx.x;
    const int ys = a.row_begin + (blockIdx.y * BY + threadIdx.y) * RY;
    if (ys >= a.row_end) return;
    const int ye = min(ys + RY, a.row_end);
    const float c[5] = {a.fparam[0], a.fparam[1], a.fparam[2], a.fparam[3], a.fparam[4]};
    const size_t sb = (size_t)a.src_row_begin, db = (size_t)a.dst_row_begin;
    if ((W & 3) == 0) {
        // ---- vector path: lane owns columns cx .. cx+3 ------------------------------------
        const int cx = (blockIdx.x * 32 + lane) * 4;
        const int cxl = min(cx, W - 4);                         // clamped (lanes past the edge)
        const int base = blockIdx.x * 128;
#define ROW4(y) (reinterpret_cast<const float4 *>(tin + ((size_t)(y) - sb) * (size_t)W + cxl))
        float4 N = __ldg(ROW4(max(ys - 1, 0)));
        float4 T = __ldg(ROW4(ys));
#pragma unroll 4
        for (int y = ys; y < ye; ++y) {
            const float4 S = __ldg(ROW4(min(y + 1, H - 1)));
            const float4 P = __ldg(reinterpret_cast<const float4 *>(pw + ((size_t)y - sb) * (size_t)W + cxl));
            float Wv = __shfl_up_sync(0xffffffffu, T.w, 1);
            float Ev = __shfl_down_sync(0xffffffffu, T.x, 1);
            const float *trow = tin + ((size_t)y - sb) * (size_t)W;
            if (lane == 0) Wv = (base == 0) ? T.x : __ldg(trow + base - 1);
            if (lane == 31) Ev = (base + 128 >= W) ? T.w : __ldg(trow + base + 128);
            if (cx + 4 >= W) Ev = T.w;                          // clamp at the east edge
            if (cx == 0) Wv = T.x;                              // clamp at the west edge
            float4 o;   // scalar: this HBM-bound one-step kernel measured 9 % slower with hs_cell4
            o.x = hs_cell(T.x, N.x, S.x, T.y, Wv, P.x, c);
            o.y = hs_cell(T.y, N.y, S.y, T.z, T.x, P.y, c);
            o.z = hs_cell(T.z, N.z, S.z, T.w, T.y, P.z, c);
            o.w = hs_cell(T.w, N.w, S.w, Ev, T.z, P.w, c);
            if (cx < W) *reinterpret_cast<float4 *>(tout + ((size_t)y - db) * (size_t)W + cx) = o;
            N = T;
            T = S;
        }
#undef ROW4
    } else {
        // ---- scalar path (rows not 16-byte aligned): lane owns 4 strided columns ---------
#pragma unroll 1
        for (int k = 0; k < 4; ++k) {
            const int xr = blockIdx.x * 128 + k * 32 + lane;
            const int x = min(xr, W - 1);
            const float *col = tin + x;
            float N = __ldg(col + ((size_t)max(ys - 1, 0) - sb) * (size_t)W);
            float T = __ldg(col + ((size_t)ys - sb) * (size_t)W);
#pragma unroll 1
            for (int y = ys; y < ye; ++y) {
                const float *trow = tin + ((size_t)y - sb) * (size_t)W;
                const float S = __ldg(col + ((size_t)min(y + 1, H - 1) - sb) * (size_t)W);
                const float P = __ldg(pw + ((size_t)y - sb) * (size_t)W + x);
                const float Wv = __ldg(trow + max(x - 1, 0));
                const float Ev = __ldg(trow + min(x + 1, W - 1));
                const float o = hs_cell(T, N, S, Ev, Wv, P, c);
                if (xr < W) tout[((size_t)y - db) * (size_t)W + xr] = o;
                N = T;
                T = S;
            }
        }
    }
}

// T = 256 threads (32 x 8 warps): 128 columns x 8 strips of 16 rows per CTA.
extern "C" __global__ void __launch_bounds__(256) orion_hotspot_f32_256(orion_kargs a) { ORION_PROBE(a); hotspot_body<8, 16>(a); }
// T = 128 threads (32 x 4 warps): 128 columns x 4 strips of 16 rows per CTA.
extern "C" __global__ void __launch_bounds__(128) orion_hotspot_f32_128(orion_kargs a) { ORION_PROBE(a); hotspot_body<4, 16>(a); }

// ---- temporal blocking: rows streamed through a shared-memory ring ------------------------
// A warp's T0 / P rows are fetched ahead with cp.async (LDGSTS: global -> shared without
// registers), so the bytes in flight per SM do not depend on the register budget of the
// occupancy level.  Each lane copies its own 16 bytes of a row into its warp's ring slot and
// later reads back exactly what it copied: no warp barrier is needed.
#ifndef H2_ROWS
#define H2_ROWS 32
#endif

__device__ __forceinline__ void cp_async16(float *sdst, const float *gsrc)
{
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"((unsigned)__cvta_generic_to_shared(sdst)),
                 "l"(gsrc) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;\n" ::"n"(N) : "memory"); }


// ---- two steps per launch, halo lanes (hotspot2h) ------------------------------------------
// The same two-step update with the warp's column halo carried by whole lanes instead of edge
// lanes: a warp loads 128 consecutive columns [base-4, base+124) as float4 lanes and writes the
// 120 columns [base, base+120) of lanes 1..30.  Lane 0's last and lane 31's first T1 cells are
// exactly the step-1 halo the outer T2 cells need (their own neighbours are in-lane or one
// shuffle away), so there are no scalar outer-column loads, no extra T1 cell and no per-lane
// edge copies: per row two 16-byte cp.async, two 16-byte ring reads, four shuffles.  6.7 % of
// the lanes' cells are recomputed halo (the neighbouring warp's), traded for half the
// memory-pipe instructions of an edge-lane form (round 1's hotspot2_f32, measured 0.142 vs
// 0.140 ms and removed).  Clamp-to-edge: the lane holding column 0 takes
// its own value as W, the lane holding column W-1 its own value as E; lanes past either edge
// load clamped columns, write nothing and feed no written cell.  Bit-identical to one-step
// launches (every cell is hs_cell4's operation sequence, = hs_cell's).
namespace {
constexpr int H2H_NB = 6;                   // ring slots per warp: the 6-row body's static slots
constexpr int H2H_SLOT = 256;               // floats: T0 segment (128) + P segment (128)
}  // namespace

template <int RY, bool BOTTOM>
__device__ __forceinline__ void hotspot2h_strip(const orion_kargs &a, int ys, int ye)
{
    extern __shared__ float4 smem4[];
    const int W = a.width, H = a.height;
    const int lane = threadIdx.x;
    const float c[5] = {a.fparam[0], a.fparam[1], a.fparam[2], a.fparam[3], a.fparam[4]};
    const int base = blockIdx.x * 120;
    const int cx = base - 4 + 4 * lane;            // the lane's first column (lane 0: halo)
    const int cxl = clampi(cx, 0, W - 4);
    const bool writer = lane >= 1 && lane <= 30 && cx < W;
    const bool wclamp = cx == 0, eclamp = cx + 4 >= W;
    const float *t0 = (const float *)a.src - (size_t)a.src_row_begin * (size_t)W;
    const float *p0 = (const float *)a.aux - (size_t)a.src_row_begin * (size_t)W;
    float *ring = reinterpret_cast<float *>(smem4) + threadIdx.y * (H2H_NB * H2H_SLOT);
    const int own = 4 * lane;

    auto step = [&c, wclamp, eclamp](const float4 &N, const float4 &T, const float4 &S, const float4 &P) {
        float Wv = __shfl_up_sync(0xffffffffu, T.w, 1);
        float Ev = __shfl_down_sync(0xffffffffu, T.x, 1);
        if (wclamp) Wv = T.x;
        if (eclamp) Ev = T.w;
        return hs_cell4(T, N, S, Ev, Wv, P, c);
    };
    auto rowp = [&](const float *b, int y) { return b + (size_t)clampi(y, 0, H - 1) * (size_t)W + cxl; };
    auto load = [&](const float *p) { return __ldg(reinterpret_cast<const float4 *>(p)); };
    // issue() runs for q = 0, 1, ... in order: slot q % NB gets T0(clamp(ys+2+q)) and P(ys+1+q)
    const float *tn = rowp(t0, ys + 2), *pn = rowp(p0, ys + 1);
    int rt = ys + 2;
    auto issue = [&](float *sl) {
        cp_async16(sl + own, tn);
        cp_async16(sl + 128 + own, pn);
        if (!BOTTOM || rt < H - 1) tn += W;
        pn += W;
        ++rt;
    };
    const int yb = min(ye, H - 1);
    const int nq = yb - ys;
#pragma unroll
    for (int q = 0; q < H2H_NB - 1; ++q) {
        if (q < nq) issue(ring + q * H2H_SLOT);
        cp_async_commit();
    }
    const bool top = ys == 0;
    const float4 tm2 = load(rowp(t0, ys - 2)), tm1 = load(rowp(t0, ys - 1));
    float4 tc0 = load(rowp(t0, ys)), tc1 = load(rowp(t0, ys + 1)), tcx;
    const float4 Pa = load(rowp(p0, ys - 1));
    float4 pa = load(rowp(p0, ys)), pb;
    float4 ua = top ? step(tc0, tc0, tc1, pa) : step(tm2, tm1, tc0, Pa);
    float4 ub = step(tm1, tc0, tc1, pa), uz;
    float *orow = (float *)a.dst + (size_t)cx + ((size_t)ys - (size_t)a.dst_row_begin) * (size_t)W;
    auto row = [&](int q, const float *sl_read, float *sl_issue, const float4 &A, const float4 &B, float4 &C,
                   const float4 &X, const float4 &Y, float4 &Z, const float4 &Pcur, float4 &Pnext) {
        if (q + H2H_NB - 1 < nq) issue(sl_issue);
        cp_async_commit();
        cp_async_wait<H2H_NB - 1>();
        C = *reinterpret_cast<const float4 *>(sl_read + own);
        Pnext = *reinterpret_cast<const float4 *>(sl_read + 128 + own);
        Z = step(A, B, C, Pnext);                  // T1(y+1)
        const float4 o = step(X, Y, Z, Pcur);      // T2(y)
        if (writer) *reinterpret_cast<float4 *>(orow) = o;
        orow += W;
    };
    int q = 0;
#define H2H_S(k) (ring + (k) * H2H_SLOT)
#define H2H_I(k) H2H_S(((k) + H2H_NB - 1) % H2H_NB)
#pragma unroll 1
    for (; q + 6 <= nq; q += 6) {                  // slot of row q + k is k
        row(q, H2H_S(0), H2H_I(0), tc0, tc1, tcx, ua, ub, uz, pa, pb);
        row(q + 1, H2H_S(1), H2H_I(1), tc1, tcx, tc0, ub, uz, ua, pb, pa);
        row(q + 2, H2H_S(2), H2H_I(2), tcx, tc0, tc1, uz, ua, ub, pa, pb);
        row(q + 3, H2H_S(3), H2H_I(3), tc0, tc1, tcx, ua, ub, uz, pb, pa);
        row(q + 4, H2H_S(4), H2H_I(4), tc1, tcx, tc0, ub, uz, ua, pa, pb);
        row(q + 5, H2H_S(5), H2H_I(5), tcx, tc0, tc1, uz, ua, ub, pb, pa);
    }
#pragma unroll 1
    for (; q < nq; ++q) {
        row(q, H2H_S(q % H2H_NB), H2H_I(q % H2H_NB), tc0, tc1, tcx, ua, ub, uz, pa, pb);
        tc0 = tc1;
        tc1 = tcx;
        ua = ub;
        ub = uz;
        pa = pb;
    }
#undef H2H_S
#undef H2H_I
    cp_async_wait<0>();
    if (ye == H) {
        const float4 o = step(ua, ub, ub, pa);
        if (writer) *reinterpret_cast<float4 *>(orow) = o;
    }
}

// T = 256 threads (32 x 8 warps): 120 output columns x 8 strips of H2_ROWS rows per CTA.
extern "C" __global__ void __launch_bounds__(256) orion_hotspot2h_f32_256(orion_kargs a)
{
    ORION_PROBE(a);
    const int ys = a.row_begin + (blockIdx.y * 8 + threadIdx.y) * H2_ROWS;
    if (ys >= a.row_end) return;
    const int ye = min(ys + H2_ROWS, a.row_end);
    if (ye + 1 < a.height)
        hotspot2h_strip<H2_ROWS, false>(a, ys, ye);
    else
        hotspot2h_strip<H2_ROWS, true>(a, ys, ye);
}

// ---- S steps per launch, halo lanes (hotspot4h: S = 4) -------------------------------------
// hotspot2h's layout carried to S <= 4 steps: a warp loads 128 consecutive columns
// [base-4, base+124) as float4 lanes and writes the 120 columns of lanes 1..30.  Step s's valid
// columns shrink by one per side per step and lanes 0 / 31 hold 4 halo columns each, so 4 steps
// fit.  Vertically the warp walks its strip of HS_ROWS rows as a pipeline over iterations
// t = ys-S .. ye-1+S: T0 row t arrives from the ring, then step s computes its row t-s from step
// s-1's rows t-s-1 .. t-s+1 (kept in registers, 3 float4 per step; stage s only from iteration
// 2s on, earlier rows being outside what stage s+1 needs), and step S's row t-S is the output.
// Per launch the kernel reads T0 and P once and writes T_S once: 12 B of DRAM per cell for S
// cell-steps (+ S/HS_ROWS re-read halo rows).  Strips touching row 0 or H-1 take the EDGE form,
// which clamps each step's N / S neighbour at rows 0 / H-1 to the cell itself (the T0 rows
// beyond the grid are clamped loads); warps holding column 0 or W-1 take the CEDGE form (the
// clamped E / W neighbour).  Every cell is hs_cell4's operation sequence with clamp-to-edge
// neighbours: bit-identical to S one-step launches.
//
// The ring: slot q holds the T0 and P rows of iteration q, fetched D = NB-S-1 iterations ahead
// by cp.async, and lives until step S has read its P row, S iterations later, so the power rows
// need no registers.  The loop body is NB rows (NB % 3 == 0: the step windows rotate with period
// 3), so every slot offset is a compile-time constant.  Measured on C3 (8192^2, A/B on one box):
// power rows in registers 0.1599 ms per launch, from the ring 0.1559; a 12-row body 0.176
// (instruction-cache bound); 32-row strips 0.1623 (more halo recompute); odd warps walking
// upwards (halo rows read by both neighbours at the same time: 549 instead of 604 MB of DRAM
// reads) 0.1600; a 12-slot ring (7 rows in flight, 12-row body) 0.178; a 3-row body carrying
// the slot index 0.161; a persistent grid (one wave, each warp one ~240-row strip: 560 instead
// of 604 MB of DRAM reads, no partial wave) 0.1665 vs 0.1550 -- fewer DRAM bytes alone do not
// make this kernel faster; at 4 warps per scheduler it is bound by issue and latency as much as
// by DRAM (long-scoreboard 1.9 stalls per issue on the ring waits, FMA pipe 56 % busy).  64-row
// strips also make a strip's 72 iterations exactly the 9 prologue/fill iterations + 7 bodies of 9
// (no slow remainder loop): 61-row strips (3.96 instead of 3.73 waves) measured 0.159 vs 0.156.
// Round 2: the ring rows moved by TMA bulk copies (cp.async.bulk of each warp's 512-byte T0 and
// P segments by one elected lane, completing on per-slot mbarriers; edge column blocks kept
// LDGSTS) measured 0.176 vs 0.157 ms per launch (three A/B pairs on one box), and a 12-slot TMA
// ring 0.218 ms: at this granularity the per-row elect / expect_tx / try_wait / warp-sync cost
// more than the 2 LDGSTS they replace.  Removed.  128-row strips (half the halo re-reads, the same
// 0.93 wave efficiency at 8192^2) measured 0.163 vs 0.154 ms (three A/B pairs) with grid-wide waits
// between launches; with chained launches (orion_chain: no idle last wave) they measure 0.1401-
// 0.1412 vs 0.1421-0.1436 ms for 64-row strips (three A/B rounds on one box): kept.  256-row strips
// (276 CTAs, less than one wave of 296 slots) chained: 0.158 vs 0.1405 ms (three A/B pairs).
#ifndef HS_ROWS
#define HS_ROWS 128
#endif
namespace {
constexpr int HS_SLOT = 256;                // floats: T0 row segment (128) + P row segment (128)
}  // namespace

template <int S, int NB, bool EDGE, bool CEDGE>
__device__ __forceinline__ void hotspotS_strip(const orion_kargs &a, int ys, int ye)
{
    static_assert(S >= 1 && S <= 4, "one float4 halo lane per side carries at most 4 steps");
    static_assert(NB % 3 == 0 && NB - S - 1 >= 1 && 2 * S < NB, "ring: NB-S-1 rows in flight, body of NB rows");
    constexpr int D = NB - S - 1;
    extern __shared__ float4 smem4[];
    const int W = a.width, H = a.height;
    const int lane = threadIdx.x;
    const float c[5] = {a.fparam[0], a.fparam[1], a.fparam[2], a.fparam[3], a.fparam[4]};
    const int base = blockIdx.x * 120;
    const int cx = base - 4 + 4 * lane;
    const int cxl = clampi(cx, 0, W - 4);
    const bool writer = lane >= 1 && lane <= 30 && cx < W;
    const bool wclamp = cx == 0, eclamp = cx + 4 >= W;
    const float *t0 = (const float *)a.src - (size_t)a.src_row_begin * (size_t)W + cxl;
    const float *p0 = (const float *)a.aux - (size_t)a.src_row_begin * (size_t)W + cxl;
    float *ring = reinterpret_cast<float *>(smem4) + threadIdx.y * (NB * HS_SLOT) + 4 * lane;
    const int nq = (ye - ys) + 2 * S;              // iterations t = ys-S .. ye-1+S
    int rt = ys - S;                               // row of the next issue (T0 and P)
    const float *tn = t0 + (ptrdiff_t)rt * W, *pn = p0 + (ptrdiff_t)rt * W;   // interior strips
    auto issue = [&](float *sl) {
        if (EDGE) {
            const size_t o = (size_t)clampi(rt, 0, H - 1) * (size_t)W;
            cp_async16(sl, t0 + o);
            cp_async16(sl + 128, p0 + o);
            ++rt;
        } else {
            cp_async16(sl, tn);
            cp_async16(sl + 128, pn);
            tn += W;
            pn += W;
        }
    };
#pragma unroll
    for (int q = 0; q < D; ++q) {
        if (q < nq) issue(ring + q * HS_SLOT);
        cp_async_commit();
    }
    float4 X[S][3];
#pragma unroll
    for (int s = 0; s < S; ++s) X[s][0] = X[s][1] = X[s][2] = make_float4(0.f, 0.f, 0.f, 0.f);
    float *orow = (float *)a.dst + (size_t)cx + ((size_t)ys - (size_t)a.dst_row_begin) * (size_t)W;
    int t = ys - S;                                // T0 row arriving this iteration
    // iteration q, kq = q % NB (a constant inside the unrolled body), steps 1 .. smin
    auto row = [&](int q, int kq, int smin) {
        if (q + D < nq) issue(ring + ((kq + D) % NB) * HS_SLOT);
        cp_async_commit();
        cp_async_wait<D>();
        X[0][0] = X[0][1];
        X[0][1] = X[0][2];
        X[0][2] = *reinterpret_cast<const float4 *>(ring + kq * HS_SLOT);            // T0(t)
#pragma unroll
        for (int s = 1; s <= S; ++s) {
            if (s > smin) continue;
            float4 Nv = X[s - 1][0], Tv = X[s - 1][1], Sv = X[s - 1][2];             // rows t-s-1 .. t-s+1
            if (EDGE) {
                const int r = t - s;
                if (r == 0) Nv = Tv;
                if (r == H - 1) Sv = Tv;
            }
            float Wv = __shfl_up_sync(0xffffffffu, Tv.w, 1);
            float Ev = __shfl_down_sync(0xffffffffu, Tv.x, 1);
            if (CEDGE) {
                if (wclamp) Wv = Tv.x;
                if (eclamp) Ev = Tv.w;
            }
            const float4 Pv = *reinterpret_cast<const float4 *>(ring + ((kq - s + NB) % NB) * HS_SLOT + 128);
            const float4 o = hs_cell4(Tv, Nv, Sv, Ev, Wv, Pv, c);                   // T_s(t-s)
            if (s < S) {
                X[s][0] = X[s][1];
                X[s][1] = X[s][2];
                X[s][2] = o;
            } else {                                                                   // row t-S >= ys
                if (writer) *reinterpret_cast<float4 *>(orow) = o;
                orow += W;
            }
        }
        ++t;
    };
    // nq >= 2S + 1 always (a strip has >= 1 row)
#pragma unroll
    for (int q = 0; q < 2 * S; ++q) row(q, q, q / 2);
    int q = 2 * S;
#pragma unroll
    for (int k = 2 * S; k < NB; ++k, ++q)          // up to the first multiple of NB
        if (q < nq) row(q, k, S);
#pragma unroll 1
    for (; q + NB <= nq; q += NB) {
#pragma unroll
        for (int k = 0; k < NB; ++k) row(q + k, k, S);
    }
#pragma unroll 1
    for (; q < nq; ++q) row(q, q % NB, S);
    cp_async_wait<0>();
    if (a.nfan) {
        // halo exchange of a row-sharded grid (off the hot loop): the band's first S and last S output
        // rows -- the halos the neighbouring bands' next launch reads -- go from dst (written above
        // by this same lane) into fan[0] / fan[1] (the upper / lower neighbour's next input, global
        // row y at y * W; NULL at the grid's edge), over NVLink when those are peer buffers
        const float *ob = (const float *)a.dst + (size_t)cx - (size_t)a.dst_row_begin * (size_t)W;
        if (writer && a.fan[0])
            for (int y = max(ys, a.row_begin); y < min(ye, a.row_begin + S); ++y)
                *reinterpret_cast<float4 *>((float *)a.fan[0] + (size_t)y * (size_t)W + cx) =
                    *reinterpret_cast<const float4 *>(ob + (size_t)y * (size_t)W);
        if (writer && a.fan[1])
            for (int y = max(ys, a.row_end - S); y < ye; ++y)
                *reinterpret_cast<float4 *>((float *)a.fan[1] + (size_t)y * (size_t)W + cx) =
                    *reinterpret_cast<const float4 *>(ob + (size_t)y * (size_t)W);
    }
}

// A chained launch (orion_chain) waits for the previous launch's 3 x 3 neighbourhood of tiles --
// every tile whose output rows / columns this CTA's strips read (halo S <= 4 < the 120 x 512
// tile) or whose input this CTA's output overwrites (ping-pong) -- instead of the whole grid.
template <int S, int RY, int NB>
__device__ __forceinline__ void hotspotS_body(const orion_kargs &a)
{
    const bool chained = a.chain != nullptr;
    if (chained) chain_wait(a, 1, 0, 1, 0);
    const int ys = a.row_begin + (blockIdx.y * 8 + threadIdx.y) * RY;
    if (ys < a.row_end) {
        const int ye = min(ys + RY, a.row_end);
        const bool redge = ys - S < 0 || ye - 1 + S > a.height - 1;
        const bool cedge = blockIdx.x == 0 || (int)blockIdx.x * 120 + 124 >= a.width;
        if (!redge && !cedge)
            hotspotS_strip<S, NB, false, false>(a, ys, ye);
        else
            hotspotS_strip<S, NB, true, true>(a, ys, ye);
    }
    if (chained) chain_signal(a);
}

// T = 256 threads (32 x 8 warps): 120 output columns x 8 strips of HS_ROWS rows per CTA; 4 steps
// per launch, 9-slot ring (4 rows in flight) per warp.
extern "C" __global__ void __launch_bounds__(256) orion_hotspot4h_f32_256(orion_kargs a)
{
    ORION_PROBE(a);
    hotspotS_body<4, HS_ROWS, 9>(a);
}
