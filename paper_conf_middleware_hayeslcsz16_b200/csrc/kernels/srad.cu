// srad.cu -- SRAD, speckle-reducing anisotropic diffusion (Table 2 P:L739,
// Fig. 10 P:L657-L693 -- the paper's downward-tuning example: half occupancy gives the
// same runtime).  Update rule per DESIGN.md reading R-SRAD (Rodinia srad_v2, ref [6]):
//   q0sqr = var(J_ROI) / mean(J_ROI)^2                       (orion_srad_roi_stats)
//   dN.. = neighbour - J;  G2 = sum d^2 / J^2;  L = sum d / J
//   qsqr = (G2/2 - L^2/16) / (1 + L/4)^2
//   c = 1 / (1 + (qsqr - q0sqr) / (q0sqr (1 + q0sqr))), clamped to [0, 1]
//   J' = J + lambda/4 * (c dN + c_S dS + c dW + c_E dE)
// Clamp-to-edge neighbours.  One iteration = the ROI statistics kernel (one CTA, a
// deterministic fixed-order double reduction) + the tunable update kernel.
//
// fp32 evaluation (reading R-SRAD-FP): multiplying numerator and denominator of qsqr by
// J^2 gives the same quantity with ONE reciprocal,
//   qsqr = (sum d^2 / 2 - (sum d)^2 / 16) / (J + sum d / 4)^2,
// and the two reciprocals left are MUFU.RCP (rcp.approx.ftz, <= 1 ulp) instead of IEEE
// divisions; products feeding sums are FFMA.  The operation sequence is fixed in
// srad_coeff / srad_update below (explicit .rn intrinsics, PTX built with -fmad=false),
// so every kernel of this file and every occupancy variant is bit-identical; the oracle
// (double, Rodinia's order) is matched to the tolerance the tests state.
#include "common.cuh"

namespace {

ORION_DEVICE float rcp_approx(float x)
{
    float y;
    asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}

// The coefficient of a cell and the differences its own update reuses.
struct SradCell {
    float c;     // diffusion coefficient, in [0, 1]
    float dnw;   // dN + dW
    float ds, de;
};

// q0 = q0sqr; nq = -q0sqr * iqden; iqden = 1 / (q0sqr (1 + q0sqr)) (launch-uniform).
ORION_DEVICE SradCell srad_coeff(float Jc, float N, float S, float Wv, float E, float iqden, float nq)
{
    const float dN = __fsub_rn(N, Jc), dS = __fsub_rn(S, Jc);
    const float dW = __fsub_rn(Wv, Jc), dE = __fsub_rn(E, Jc);
    const float g2 = __fmaf_rn(dE, dE, __fmaf_rn(dW, dW, __fmaf_rn(dS, dS, __fmul_rn(dN, dN))));
    const float dnw = __fadd_rn(dN, dW);
    const float sd = __fadd_rn(__fadd_rn(dnw, dS), dE);
    // 16*num and 4*den: power-of-two scalings commute with every rounding below, so
    // qsqr = (16 num) * rcp(16 den^2) is bit-identical to num * rcp(den^2), one FMUL less
    const float num16 = __fmaf_rn(-sd, sd, __fmul_rn(8.0f, g2));
    const float den4 = __fmaf_rn(4.0f, Jc, sd);
    const float qsqr = __fmul_rn(num16, rcp_approx(__fmul_rn(den4, den4)));
    const float c = rcp_approx(__fadd_rn(1.0f, __fmaf_rn(qsqr, iqden, nq)));
    SradCell r;
    r.c = __saturatef(c);
    r.dnw = dnw;
    r.ds = dS;
    r.de = dE;
    return r;
}

// J' = J + lambda/4 * (c (dN + dW) + c_S dS + c_E dE)
ORION_DEVICE float srad_update(float Jc, const SradCell &k, float cS, float cE, float lam4)
{
    return __fmaf_rn(lam4, __fmaf_rn(k.c, k.dnw, __fmaf_rn(cS, k.ds, __fmul_rn(cE, k.de))), Jc);
}

// The same two functions for a pair of horizontally adjacent cells on the packed fp32x2 pipe
// (FADD2 / FMUL2 / FFMA2: two independent IEEE .rn operations per instruction, bit-identical
// to the scalar forms above, operation by operation).  dW / dE of a pair are not register
// pairs of the row, so they are scalar FSUBs written straight into pairs; every other step is
// one packed instruction for both cells.
struct SradPair {
    float2 c, dnw, ds, de;
};
ORION_DEVICE float2 f2(float v) { return make_float2(v, v); }
ORION_DEVICE float2 neg(float2 v) { return make_float2(-v.x, -v.y); }
ORION_DEVICE SradPair srad_coeff2(float2 Jc, float2 N, float2 S, float2 dW, float2 dE, float iqden, float nq)
{
    const float2 dN = __fadd2_rn(N, neg(Jc)), dS = __fadd2_rn(S, neg(Jc));
    const float2 g2 = __ffma2_rn(dE, dE, __ffma2_rn(dW, dW, __ffma2_rn(dS, dS, __fmul2_rn(dN, dN))));
    const float2 dnw = __fadd2_rn(dN, dW);
    const float2 sd = __fadd2_rn(__fadd2_rn(dnw, dS), dE);
    const float2 num16 = __ffma2_rn(neg(sd), sd, __fmul2_rn(f2(8.0f), g2));   // as srad_coeff
    const float2 den4 = __ffma2_rn(f2(4.0f), Jc, sd);
    const float2 dd = __fmul2_rn(den4, den4);
    const float2 qsqr = __fmul2_rn(num16, make_float2(rcp_approx(dd.x), rcp_approx(dd.y)));
    const float2 t = __fadd2_rn(f2(1.0f), __ffma2_rn(qsqr, f2(iqden), f2(nq)));
    SradPair r;
    r.c = make_float2(__saturatef(rcp_approx(t.x)), __saturatef(rcp_approx(t.y)));
    r.dnw = dnw;
    r.ds = dS;
    r.de = dE;
    return r;
}
ORION_DEVICE float2 srad_update2(float2 Jc, const SradPair &k, float2 cS, float2 cE, float lam4)
{
    return __ffma2_rn(f2(lam4), __ffma2_rn(k.c, k.dnw, __ffma2_rn(cS, k.ds, __fmul2_rn(cE, k.de))), Jc);
}

struct SradConsts {
    float lam4, iqden, nq;
};

ORION_DEVICE SradConsts srad_consts(const orion_kargs &a)
{
    const float q0 = *(const float *)a.aux;
    SradConsts k;
    k.lam4 = __fmul_rn(0.25f, a.fparam[0]);
    k.iqden = __frcp_rn(__fmul_rn(q0, __fadd_rn(1.0f, q0)));
    k.nq = -__fmul_rn(q0, k.iqden);
    return k;
}

// ---- ROI statistics carried by the grids (srad_f32hs) ------------------------------------------
// The fused kernel reads q0sqr of ITS input from partial sums stored behind the input grid and
// writes the partial sums of its output's ROI behind the output grid, so the next iteration needs
// no separate statistics kernel.  Partition (shared with orion_srad_stats_init): the warp
// (strip g = y / SRADH_RY, column block b = x / 120) owning a ROI cell sums, in double, the ROI
// cells it writes -- each lane its own columns row by row, then a fixed xor-shuffle tree -- into
// slot (g - g1) * nb + (b - b1), g1 / b1 the first strip / block the ROI touches.  Every launch
// reduces the slots in index order, so q0sqr is deterministic and the same at every level.
#ifndef SRADH_RY
#define SRADH_RY 42
#endif
constexpr int SRAD_STAT_SLOTS = 64;           // (sum, sum of squares) doubles per slot

struct SradRoi {
    int r1, r2, c1, c2;      // inclusive ROI
    int g1, b1, nb, nslots;  // first strip / block, blocks per strip row, slots used
};
ORION_DEVICE SradRoi srad_roi(const orion_kargs &a)
{
    SradRoi r;
    r.r1 = (int)a.fparam[1];
    r.r2 = (int)a.fparam[2];
    r.c1 = (int)a.fparam[3];
    r.c2 = (int)a.fparam[4];
    r.g1 = r.r1 / SRADH_RY;
    r.b1 = r.c1 / 120;
    r.nb = r.c2 / 120 - r.b1 + 1;
    r.nslots = (r.r2 / SRADH_RY - r.g1 + 1) * r.nb;
    return r;
}
// The statistics area behind a width x height grid (16-byte aligned: width % 4 == 0).
ORION_DEVICE double *srad_stats_area(const void *grid, const orion_kargs &a, int row_begin)
{
    return (double *)((float *)grid + ((size_t)a.height - (size_t)row_begin) * (size_t)a.width);
}
// q0sqr from the slots of the input grid: lane k reduces slots k, k+32 (fixed order), then a
// fixed xor tree; every lane returns the same value.
ORION_DEVICE float srad_q0_from_slots(const double *slots, const SradRoi &r, int lane)
{
    double s = 0.0, s2 = 0.0;
    for (int k = lane; k < r.nslots; k += 32) {     // through L2 (written by other SMs, see chain_wait)
        s += __ldcg(slots + 2 * k);
        s2 += __ldcg(slots + 2 * k + 1);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        s += __shfl_xor_sync(0xffffffffu, s, o);
        s2 += __shfl_xor_sync(0xffffffffu, s2, o);
    }
    const double n = (double)(r.r2 - r.r1 + 1) * (double)(r.c2 - r.c1 + 1);
    const double mean = s / n;
    const double var = s2 / n - mean * mean;
    return (float)(var / (mean * mean));
}
ORION_DEVICE SradConsts srad_consts_q0(float q0, float lam)
{
    SradConsts k;
    k.lam4 = __fmul_rn(0.25f, lam);
    k.iqden = __frcp_rn(__fmul_rn(q0, __fadd_rn(1.0f, q0)));
    k.nq = -__fmul_rn(q0, k.iqden);
    return k;
}
// A lane's running ROI sums over the float4 it holds at columns cx .. cx+3 of row y.
ORION_DEVICE void srad_roi_acc(double &s, double &s2, const float4 &v, int cx, int y, const SradRoi &r, bool own)
{
    if (!own || y < r.r1 || y > r.r2) return;
    const float e[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
    for (int k = 0; k < 4; ++k)
        if (cx + k >= r.c1 && cx + k <= r.c2) {
            const double d = (double)e[k];
            s += d;
            s2 = fma(d, d, s2);
        }
}
// Close a warp's sums: fixed xor tree, lane 0 stores its slot (warps outside the ROI store nothing).
ORION_DEVICE void srad_roi_store(double s, double s2, double *area, int g, int b, const SradRoi &r, int lane)
{
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        s += __shfl_xor_sync(0xffffffffu, s, o);
        s2 += __shfl_xor_sync(0xffffffffu, s2, o);
    }
    if (lane == 0) {
        const int k = (g - r.g1) * r.nb + (b - r.b1);
        area[2 * k] = s;
        area[2 * k + 1] = s2;
    }
}

constexpr int SX = 32, SY = 8, RY = 4;        // threads, rows per thread
constexpr int TW = SX, TH = SY * RY;          // output tile 32 x 32
constexpr int JW = TW + 3, JH = TH + 3;       // J tile: x0-1 .. x0+TW+1, y0-1 .. y0+TH+1
constexpr int CW = TW + 1, CH = TH + 1;       // c tile: x0 .. x0+TW, y0 .. y0+TH

}  // namespace

// ---- shared-memory tile kernel (cross-check form) -----------------------------------------
// CTA = 32 x 8 threads, output tile 32 x 32 cells (4 rows per thread).  The J tile with a
// 1-cell halo (+1 extra row / column south / east for the neighbours' coefficients) is
// staged in shared memory; the coefficients of the tile plus one row south and one column
// east are computed once into shared memory (the two-kernel Rodinia form writes c and four
// derivative arrays to DRAM instead); then J' is formed.
extern "C" __global__ void __launch_bounds__(256) orion_srad_f32_256(orion_kargs a)
{
    ORION_PROBE(a);
    extern __shared__ float4 smem4[];
    float *js = reinterpret_cast<float *>(smem4);   // JH x JW
    float *cs = js + JH * JW;                       // CH x CW
    const float *J = (const float *)a.src;
    const int W = a.width, H = a.height;
    const int tid = threadIdx.y * SX + threadIdx.x;
    const int x0 = blockIdx.x * TW;
    const int y0 = a.row_begin + blockIdx.y * TH;
    for (int idx = tid; idx < JW * JH; idx += SX * SY) {
        const int ty = idx / JW, tx = idx - ty * JW;
        const int gx = clampi(x0 - 1 + tx, 0, W - 1), gy = clampi(y0 - 1 + ty, 0, H - 1);
        js[idx] = __ldg(J + (size_t)(gy - a.src_row_begin) * (size_t)W + gx);
    }
    const SradConsts k = srad_consts(a);
    __syncthreads();
    // coefficient tile: cell (y0+cy, x0+cx), cy in [0, CH), cx in [0, CW).  The cell at
    // global (gy, gx) with gy >= H or gx >= W is a clamped copy: its coefficient is the
    // edge cell's, which the clamped J values reproduce (all its neighbours clamp alike).
    auto tile_cell = [&](int gy, int gx) {
        const int ty = min(gy, H - 1) - (y0 - 1), tx = min(gx, W - 1) - (x0 - 1);
        const int tn = max(min(gy, H - 1) - 1, 0) - (y0 - 1), ts = min(min(gy, H - 1) + 1, H - 1) - (y0 - 1);
        const int tw = max(min(gx, W - 1) - 1, 0) - (x0 - 1), te = min(min(gx, W - 1) + 1, W - 1) - (x0 - 1);
        return srad_coeff(js[ty * JW + tx], js[tn * JW + tx], js[ts * JW + tx], js[ty * JW + tw], js[ty * JW + te],
                          k.iqden, k.nq);
    };
    for (int idx = tid; idx < CW * CH; idx += SX * SY) {
        const int cy = idx / CW, cx = idx - cy * CW;
        cs[idx] = tile_cell(y0 + cy, x0 + cx).c;
    }
    __syncthreads();
    const int cx = threadIdx.x, gx = x0 + cx;
    if (gx >= W) return;
#pragma unroll
    for (int r = 0; r < RY; ++r) {
        const int cy = threadIdx.y * RY + r, gy = y0 + cy;
        if (gy >= a.row_end) return;
        const SradCell kc = tile_cell(gy, gx);
        const float Jc = js[(gy - (y0 - 1)) * JW + (gx - (x0 - 1))];
        const float cS = cs[(min(gy + 1, H - 1) - y0) * CW + cx];
        const float cE = cs[cy * CW + (min(gx + 1, W - 1) - x0)];
        ((float *)a.dst)[(size_t)(gy - a.dst_row_begin) * (size_t)W + gx] = srad_update(Jc, kc, cS, cE, k.lam4);
    }
}

// ROI statistics: one CTA of 1024 threads; thread t sums elements t, t+1024, ... of the
// row-major ROI in double (16 loads in flight: the default 128 x 128 ROI is one batch, one
// memory latency), then a fixed-shape shuffle tree per warp and
// across the 32 warp sums -- deterministic, so every occupancy variant of the update kernel
// sees the same q0sqr.
extern "C" __global__ void __launch_bounds__(1024) orion_srad_stats(const float *J, int W, int r1, int r2, int c1,
                                                                     int c2, float *q0)
{
    __shared__ double s1[32], s2[32];
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");   // PDL (see orion_probe)
    asm volatile("griddepcontrol.wait;" ::: "memory");
    const int t = threadIdx.x;
    const int rw = c2 - c1 + 1, n = (r2 - r1 + 1) * rw;
    double a = 0.0, b = 0.0;
#pragma unroll 16
    for (int e = t; e < n; e += 1024) {
        const int i = r1 + e / rw, j = c1 + e % rw;
        const double v = __ldg(J + (size_t)i * (size_t)W + j);
        a += v;
        b += v * v;
    }
#pragma unroll
    for (int s = 16; s > 0; s >>= 1) {
        a += __shfl_down_sync(0xffffffffu, a, s);
        b += __shfl_down_sync(0xffffffffu, b, s);
    }
    if ((t & 31) == 0) {
        s1[t >> 5] = a;
        s2[t >> 5] = b;
    }
    __syncthreads();
    if (t < 32) {
        a = s1[t];
        b = s2[t];
#pragma unroll
        for (int s = 16; s > 0; s >>= 1) {
            a += __shfl_down_sync(0xffffffffu, a, s);
            b += __shfl_down_sync(0xffffffffu, b, s);
        }
        if (t == 0) {
            const double mean = a / n;
            const double var = b / n - mean * mean;
            *q0 = (float)(var / (mean * mean));
        }
    }
}

// ---- register-sliding kernel (the default srad_f32) ------------------------------------------
// A warp owns 32*V consecutive columns from x0 (V = 4: float4 lanes, 16-byte loads / stores,
// width % 4 == 0; V = 1: scalar lanes for any width), of which lanes 0..30 write their cells
// and lane 31 only supplies the coefficient lane 30's last cell needs as c_E (31V output
// columns per warp: 3 % of the arithmetic instead of a divergent extra cell).  It walks a strip
// of rows top to bottom with J rows y .. y+2 and the coefficient row y in registers, the next
// three rows in flight through a cp.async ring in shared memory (4 slots per warp, 16.9 KB
// per CTA): every J row is read once per strip, every coefficient computed once.
// W / E neighbours come by shuffle; lane 0 fetches column x0-1, lane 31 column x0+32V.
// CTA = 8 warps over a 124 x 128 tile: V = 4 -> 8 strips of 16 rows; V = 1 -> 4 column
// groups of 31 x 2 strips of 64 rows.
namespace {
constexpr int SRAD_NB = 6;      // ring slots per warp (a multiple of the 6-row loop body: static slots)
constexpr int SRAD_SLOT = 132;  // floats per slot: 32 lanes x up to 4 columns + 2 outer columns (+pad)
}  // namespace

__device__ __forceinline__ void srad_cp16(float *sdst, const float *gsrc)
{
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"((unsigned)__cvta_generic_to_shared(sdst)),
                 "l"(gsrc) : "memory");
}
__device__ __forceinline__ void srad_cp4(float *sdst, const float *gsrc)
{
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;\n" ::"r"((unsigned)__cvta_generic_to_shared(sdst)),
                 "l"(gsrc) : "memory");
}
__device__ __forceinline__ void srad_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
template <int N>
__device__ __forceinline__ void srad_wait() { asm volatile("cp.async.wait_group %0;\n" ::"n"(N) : "memory"); }

namespace {
template <int V>
struct SRow {
    float v[V];
    float xa;   // lane 0: J[max(x0-1, 0)]; lane 31: J[min(x0+32V, W-1)]; others: unused
};
template <int V>
struct CRow {
    SradCell k[V];
};
template <>
struct CRow<4> {
    SradPair p[2];   // cells (0, 1) and (2, 3)
};
}  // namespace

template <int V>
__device__ __forceinline__ void srad_strip(const orion_kargs &a, int x0, int ys, int ye)
{
    const int W = a.width, H = a.height;
    const int lane = threadIdx.x;
    const int cx = x0 + V * lane;
    const int cxl = min(cx, W - V);
    const bool east_clamp = cx + V >= W;      // the lane's last cell is the image's last column
    const bool writer = lane < 31 && cx < W;
    const SradConsts kc = srad_consts(a);
    const int xa = lane == 0 ? max(x0 - 1, 0) : (lane == 31 ? min(x0 + 32 * V, W - 1) : cxl);
    const float *J = (const float *)a.src - (size_t)a.src_row_begin * (size_t)W;   // global row 0
    float *Jo = (float *)a.dst + (size_t)cx - (size_t)a.dst_row_begin * (size_t)W;

    auto load = [&](const float *row) {
        SRow<V> r;
        if constexpr (V == 4) {
            const float4 q = __ldg(reinterpret_cast<const float4 *>(row + cxl));
            r.v[0] = q.x;
            r.v[1] = q.y;
            r.v[2] = q.z;
            r.v[3] = q.w;
        } else {
            r.v[0] = __ldg(row + cxl);
        }
        r.xa = __ldg(row + xa);
        return r;
    };
    auto coeff_row = [&](const SRow<V> &N, const SRow<V> &T, const SRow<V> &S) {
        float Wv = __shfl_up_sync(0xffffffffu, T.v[V - 1], 1);
        float Ev = __shfl_down_sync(0xffffffffu, T.v[0], 1);
        if (lane == 0) Wv = T.xa;
        if (lane == 31) Ev = T.xa;
        if (east_clamp) Ev = T.v[V - 1];
        CRow<V> c;
        if constexpr (V == 4) {
            const float *t = T.v;
            c.p[0] = srad_coeff2(make_float2(t[0], t[1]), make_float2(N.v[0], N.v[1]), make_float2(S.v[0], S.v[1]),
                                 make_float2(__fsub_rn(Wv, t[0]), __fsub_rn(t[0], t[1])),
                                 make_float2(__fsub_rn(t[1], t[0]), __fsub_rn(t[2], t[1])), kc.iqden, kc.nq);
            c.p[1] = srad_coeff2(make_float2(t[2], t[3]), make_float2(N.v[2], N.v[3]), make_float2(S.v[2], S.v[3]),
                                 make_float2(__fsub_rn(t[1], t[2]), __fsub_rn(t[2], t[3])),
                                 make_float2(__fsub_rn(t[3], t[2]), __fsub_rn(Ev, t[3])), kc.iqden, kc.nq);
        } else {
#pragma unroll
            for (int k = 0; k < V; ++k)
                c.k[k] = srad_coeff(T.v[k], N.v[k], S.v[k], k == 0 ? Wv : T.v[k - 1], k == V - 1 ? Ev : T.v[k + 1],
                                    kc.iqden, kc.nq);
        }
        return c;
    };
    auto update_row = [&](int y, const SRow<V> &T, const CRow<V> &c0, const CRow<V> &c1) {
        float o[V];
        if constexpr (V == 4) {
            float cE = __shfl_down_sync(0xffffffffu, c0.p[0].c.x, 1);
            if (east_clamp) cE = c0.p[1].c.y;
            const float2 lo = srad_update2(make_float2(T.v[0], T.v[1]), c0.p[0], c1.p[0].c,
                                           make_float2(c0.p[0].c.y, c0.p[1].c.x), kc.lam4);
            const float2 hi = srad_update2(make_float2(T.v[2], T.v[3]), c0.p[1], c1.p[1].c,
                                           make_float2(c0.p[1].c.y, cE), kc.lam4);
            o[0] = lo.x;
            o[1] = lo.y;
            o[2] = hi.x;
            o[3] = hi.y;
        } else {
            float cE = __shfl_down_sync(0xffffffffu, c0.k[0].c, 1);
            if (east_clamp) cE = c0.k[V - 1].c;
#pragma unroll
            for (int k = 0; k < V; ++k)
                o[k] = srad_update(T.v[k], c0.k[k], c1.k[k].c, k == V - 1 ? cE : c0.k[k + 1].c, kc.lam4);
        }
        if (writer) {
            float *orow = Jo + (size_t)y * (size_t)W;
            if constexpr (V == 4)
                *reinterpret_cast<float4 *>(orow) = make_float4(o[0], o[1], o[2], o[3]);
            else
                *orow = o[0];
        }
    };

    // rows y+2, y+3, ... stream through the warp's ring of SRAD_NB slots in shared memory
    // (cp.async, SRAD_NB-1 rows in flight without holding registers); slot q holds
    // J(clamp(ys+2+q)).  Each lane reads back exactly the words it copied.
    extern __shared__ float4 srad_ring4[];
    float *ring = reinterpret_cast<float *>(srad_ring4) + threadIdx.y * (SRAD_NB * SRAD_SLOT);
    const int own = V * lane, oxa = 32 * V + (lane == 0 ? 0 : 1);
    const float *pn = J + (size_t)min(ys + 2, H - 1) * (size_t)W;
    int rn = ys + 2;                                            // row pn points at (unclamped)
    auto issue = [&](float *sl) {
        if constexpr (V == 4)
            srad_cp16(sl + own, pn + cxl);
        else
            srad_cp4(sl + own, pn + cxl);
        if (lane == 0 || lane == 31) srad_cp4(sl + oxa, pn + xa);
        if (rn < H - 1) pn += W;
        ++rn;
    };
    auto slot_row = [&](const float *sl) {
        SRow<V> r;
        if constexpr (V == 4) {
            const float4 t = *reinterpret_cast<const float4 *>(sl + own);
            r.v[0] = t.x;
            r.v[1] = t.y;
            r.v[2] = t.z;
            r.v[3] = t.w;
        } else {
            r.v[0] = sl[own];
        }
        r.xa = (lane == 0 || lane == 31) ? sl[oxa] : 0.0f;
        return r;
    };
    const int yb = min(ye, H - 1);                              // rows with a distinct south row
    const int nq = yb - ys;
#pragma unroll
    for (int q = 0; q < SRAD_NB - 1; ++q) {
        if (q < nq) issue(ring + q * SRAD_SLOT);
        srad_commit();
    }
    SRow<V> j0 = load(J + (size_t)ys * (size_t)W), j1 = load(J + (size_t)min(ys + 1, H - 1) * (size_t)W), j2;
    CRow<V> c0 = coeff_row(load(J + (size_t)max(ys - 1, 0) * (size_t)W), j0, j1), c1;
    // one output row y = ys + q: N = J(y), T = J(y+1), S = J(y+2) (from the ring, written into
    // S), cT = c(y), cS = c(y+1) (written).  The row registers rotate through three variables and
    // the coefficient rows through two, so six consecutive rows are written out with permuted
    // arguments -- no register moves between rows.
    auto row = [&](int q, float *sl_read, float *sl_issue, const SRow<V> &N, const SRow<V> &T, SRow<V> &S,
                   const CRow<V> &cT, CRow<V> &cS) {
        if (q + SRAD_NB - 1 < nq) issue(sl_issue);
        srad_commit();
        srad_wait<SRAD_NB - 1>();
        S = slot_row(sl_read);
        cS = coeff_row(N, T, S);
        update_row(ys + q, N, cT, cS);
    };
    int q = 0;
#pragma unroll 1
#define SR_S(k) (ring + (k) * SRAD_SLOT)
#define SR_I(k) SR_S(((k) + SRAD_NB - 1) % SRAD_NB)
    for (; q + 6 <= nq; q += 6) {                               // slot of row q + k is k
        row(q, SR_S(0), SR_I(0), j0, j1, j2, c0, c1);
        row(q + 1, SR_S(1), SR_I(1), j1, j2, j0, c1, c0);
        row(q + 2, SR_S(2), SR_I(2), j2, j0, j1, c0, c1);
        row(q + 3, SR_S(3), SR_I(3), j0, j1, j2, c1, c0);
        row(q + 4, SR_S(4), SR_I(4), j1, j2, j0, c0, c1);
        row(q + 5, SR_S(5), SR_I(5), j2, j0, j1, c1, c0);
    }
#pragma unroll 1
    for (; q < nq; ++q) {                                       // the last < 6 rows
        row(q, SR_S(q % SRAD_NB), SR_I(q % SRAD_NB), j0, j1, j2, c0, c1);
        j0 = j1;
        j1 = j2;
        c0 = c1;
    }
#undef SR_S
#undef SR_I
    srad_wait<0>();
    if (ye == H) update_row(H - 1, j0, c0, c0);               // last image row: c_S = own c
}

// T = 256 threads (32 x 8 warps), output tile 124 x (8 * SRAD_RY).  Longer strips amortise the
// strip prologue (three J rows and one coefficient row computed before the first output row).
#ifndef SRAD_RY
#define SRAD_RY 32
#endif
extern "C" __global__ void __launch_bounds__(256) orion_srad4_f32_256(orion_kargs a)
{
    ORION_PROBE(a);
    const int w = threadIdx.y;
    if ((a.width & 3) == 0) {
        const int ys = a.row_begin + blockIdx.y * (8 * SRAD_RY) + w * SRAD_RY;
        if (ys < a.row_end) srad_strip<4>(a, blockIdx.x * 124, ys, min(ys + SRAD_RY, a.row_end));
    } else {
        const int x0 = blockIdx.x * 124 + (w & 3) * 31;
        const int ys = a.row_begin + blockIdx.y * (8 * SRAD_RY) + (w >> 2) * (4 * SRAD_RY);
        if (ys < a.row_end && x0 < a.width) srad_strip<1>(a, x0, ys, min(ys + 4 * SRAD_RY, a.row_end));
    }
}

// ---- halo-lane form (srad_f32h; width % 4 == 0) ------------------------------------------------
// The float4 strip of srad_strip<4> with the warp's column halo carried by whole lanes, as in
// hotspot2h / hotspot4h: a warp loads the 128 columns [base-4, base+124) and writes the 120
// columns of lanes 1..30.  A cell's update needs J one column west and two east (c_E needs its
// east neighbour) -- lane 0's last cell and lane 31's first cell and coefficient are exactly
// that halo -- so there are no scalar outer-column loads, no lane-0 / lane-31 branches and no
// divergent cp.async; the west / east image-edge clamps exist only in the warps that hold
// column 0 or W-1 (CEDGE).  Every cell is srad_coeff2 / srad_update2's operation sequence with
// the same clamp-to-edge neighbours: bit-identical to srad_f32 and srad_f32_tile.
namespace {
constexpr int SRADH_SLOT = 128;   // floats per ring slot: the warp's 128 columns of one J row
}  // namespace

template <bool CEDGE, bool STATS = false>
__device__ __forceinline__ void srad_strip_h(const orion_kargs &a, int base, int ys, int ye,
                                             const SradConsts *pre = nullptr)
{
    const int W = a.width, H = a.height;
    const int lane = threadIdx.x;
    const int cx = base - 4 + 4 * lane;
    const int cxl = clampi(cx, 0, W - 4);
    const bool wclamp = cx == 0, eclamp = cx + 4 >= W;
    const bool writer = lane >= 1 && lane <= 30 && cx < W;
    SradConsts kc;                  // STATS: set after the ring's first rows are in flight (below)
    if (!STATS) kc = srad_consts(a);
    const float *J = (const float *)a.src - (size_t)a.src_row_begin * (size_t)W + cxl;   // row 0, own columns
    float *Jo = (float *)a.dst + (size_t)cx - (size_t)a.dst_row_begin * (size_t)W;

    // rows written by the previous launch (possibly still running on other SMs for a chained
    // launch, orion_chain): read through L2
    auto load = [&](int y) { return __ldcg(reinterpret_cast<const float4 *>(J + (size_t)y * (size_t)W)); };
    auto coeff_row = [&](const float4 &N, const float4 &T, const float4 &S) {
        float Wv = __shfl_up_sync(0xffffffffu, T.w, 1);
        float Ev = __shfl_down_sync(0xffffffffu, T.x, 1);
        if (CEDGE) {
            if (wclamp) Wv = T.x;
            if (eclamp) Ev = T.w;
        }
        CRow<4> c;
        c.p[0] = srad_coeff2(make_float2(T.x, T.y), make_float2(N.x, N.y), make_float2(S.x, S.y),
                             make_float2(__fsub_rn(Wv, T.x), __fsub_rn(T.x, T.y)),
                             make_float2(__fsub_rn(T.y, T.x), __fsub_rn(T.z, T.y)), kc.iqden, kc.nq);
        c.p[1] = srad_coeff2(make_float2(T.z, T.w), make_float2(N.z, N.w), make_float2(S.z, S.w),
                             make_float2(__fsub_rn(T.y, T.z), __fsub_rn(T.z, T.w)),
                             make_float2(__fsub_rn(T.w, T.z), __fsub_rn(Ev, T.w)), kc.iqden, kc.nq);
        return c;
    };
    auto update_row = [&](int y, const float4 &T, const CRow<4> &c0, const CRow<4> &c1) {
        float cE = __shfl_down_sync(0xffffffffu, c0.p[0].c.x, 1);
        if (CEDGE && eclamp) cE = c0.p[1].c.y;
        const float2 lo = srad_update2(make_float2(T.x, T.y), c0.p[0], c1.p[0].c,
                                       make_float2(c0.p[0].c.y, c0.p[1].c.x), kc.lam4);
        const float2 hi = srad_update2(make_float2(T.z, T.w), c0.p[1], c1.p[1].c, make_float2(c0.p[1].c.y, cE),
                                       kc.lam4);
        if (writer) *reinterpret_cast<float4 *>(Jo + (size_t)y * (size_t)W) = make_float4(lo.x, lo.y, hi.x, hi.y);
    };

    // rows y+2, y+3, ... stream through the warp's ring (slot q holds J(clamp(ys+2+q)))
    extern __shared__ float4 srad_ring4[];
    float *ring = reinterpret_cast<float *>(srad_ring4) + threadIdx.y * (SRAD_NB * SRADH_SLOT) + 4 * lane;
    const float *pn = J + (size_t)min(ys + 2, H - 1) * (size_t)W;
    int rn = ys + 2;
    auto issue = [&](float *sl) {
        srad_cp16(sl, pn);
        if (rn < H - 1) pn += W;
        ++rn;
    };
    const int yb = min(ye, H - 1);
    const int nq = yb - ys;
#pragma unroll
    for (int q = 0; q < SRAD_NB - 1; ++q) {
        if (q < nq) issue(ring + q * SRADH_SLOT);
        srad_commit();
    }
    if (STATS)   // the input's q0sqr from its statistics slots, while the ring rows are in flight
        kc = pre ? *pre
                 : srad_consts_q0(srad_q0_from_slots(srad_stats_area(a.src, a, a.src_row_begin), srad_roi(a), lane),
                                  a.fparam[0]);
    float4 j0 = load(ys), j1 = load(min(ys + 1, H - 1)), j2;
    CRow<4> c0 = coeff_row(load(max(ys - 1, 0)), j0, j1), c1;
    auto row = [&](int q, float *sl_read, float *sl_issue, const float4 &N, const float4 &T, float4 &S,
                   const CRow<4> &cT, CRow<4> &cS) {
        if (q + SRAD_NB - 1 < nq) issue(sl_issue);
        srad_commit();
        srad_wait<SRAD_NB - 1>();
        S = *reinterpret_cast<const float4 *>(sl_read);
        cS = coeff_row(N, T, S);
        update_row(ys + q, N, cT, cS);
    };
    int q = 0;
#define SH_S(k) (ring + (k) * SRADH_SLOT)
#define SH_I(k) SH_S(((k) + SRAD_NB - 1) % SRAD_NB)
#pragma unroll 1
    for (; q + 6 <= nq; q += 6) {                               // slot of row q + k is k
        row(q, SH_S(0), SH_I(0), j0, j1, j2, c0, c1);
        row(q + 1, SH_S(1), SH_I(1), j1, j2, j0, c1, c0);
        row(q + 2, SH_S(2), SH_I(2), j2, j0, j1, c0, c1);
        row(q + 3, SH_S(3), SH_I(3), j0, j1, j2, c1, c0);
        row(q + 4, SH_S(4), SH_I(4), j1, j2, j0, c0, c1);
        row(q + 5, SH_S(5), SH_I(5), j2, j0, j1, c1, c0);
    }
#pragma unroll 1
    for (; q < nq; ++q) {
        row(q, SH_S(q % SRAD_NB), SH_I(q % SRAD_NB), j0, j1, j2, c0, c1);
        j0 = j1;
        j1 = j2;
        c0 = c1;
    }
#undef SH_S
#undef SH_I
    srad_wait<0>();
    if (ye == H) update_row(H - 1, j0, c0, c0);               // last image row: c_S = own c
    if (STATS) {
        // the output ROI's slot: a warp holding ROI cells reads back the cells its lanes just
        // wrote (same-thread global RAW; off the hot loop, so no registers live across it)
        const SradRoi roi = srad_roi(a);
        if (ys <= roi.r2 && ye - 1 >= roi.r1 && base <= roi.c2 && base + 119 >= roi.c1) {
            double rs = 0.0, rs2 = 0.0;
            for (int y = max(ys, roi.r1); y <= min(ye - 1, roi.r2); ++y)
                if (writer)
                    srad_roi_acc(rs, rs2, *reinterpret_cast<const float4 *>(Jo + (size_t)y * (size_t)W), cx, y, roi,
                                 true);
            srad_roi_store(rs, rs2, srad_stats_area(a.dst, a, a.dst_row_begin), ys / SRADH_RY, base / 120, roi, lane);
        }
    }
}

// T = 256 threads (32 x 8 warps), output tile 120 x (8 * SRADH_RY); width % 4 == 0.  42-row
// strips: a multiple of the 6-row loop body (no remainder iterations), 25 x 69 CTAs at 8192^2.
// 84-row strips (13 x 69 CTAs) measured 0.111-0.117 vs 0.0907 ms per chained iteration (three A/B pairs).
// A chained srad_f32hs launch (orion_chain) waits for the previous launch's 3 x 3 neighbourhood
// of tiles and for its ROI tiles (the writers of the statistics slots it reduces); every warp
// then reduces the slots, and only after that does the CTA let the next launch be scheduled
// (griddepcontrol.launch_dependents, dep_late): a later launch's ROI warps overwrite the slots
// behind this launch's input only once every CTA of this launch has read them.
template <bool STATS>
__device__ __forceinline__ void srad4h_body(const orion_kargs &a)
{
    const bool chained = STATS && a.chain != nullptr;
    SradConsts pre;
    if (chained) {
        const SradRoi r = srad_roi(a);
        chain_wait(a, r.c1 / 120, r.c2 / 120, r.r1 / (8 * SRADH_RY), r.r2 / (8 * SRADH_RY));
        pre = srad_consts_q0(srad_q0_from_slots(srad_stats_area(a.src, a, a.src_row_begin), r, threadIdx.x),
                             a.fparam[0]);
        __syncthreads();
        asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    }
    const int ys = a.row_begin + blockIdx.y * (8 * SRADH_RY) + threadIdx.y * SRADH_RY;
    if (ys < a.row_end) {
        const int base = blockIdx.x * 120;
        const bool cedge = base == 0 || base + 124 >= a.width;
        if (cedge)
            srad_strip_h<true, STATS>(a, base, ys, min(ys + SRADH_RY, a.row_end), chained ? &pre : nullptr);
        else
            srad_strip_h<false, STATS>(a, base, ys, min(ys + SRADH_RY, a.row_end), chained ? &pre : nullptr);
    }
    if (chained) chain_signal(a);
}
extern "C" __global__ void __launch_bounds__(256) orion_srad4h_f32_256(orion_kargs a)
{
    ORION_PROBE(a);
    srad4h_body<false>(a);
}
// srad_f32hs: the same strips with the ROI statistics fused in -- q0sqr of the input from the
// slots behind src, the output ROI's slots written behind dst (no statistics kernel per iteration).
extern "C" __global__ void __launch_bounds__(256) orion_srad4hs_f32_256(orion_kargs a)
{
    ORION_PROBE(a);
    srad4h_body<true>(a);
}

// Statistics slots of a grid J (the first iteration's input) in srad_f32hs's partition: one warp
// per (strip, block) slot of the ROI, the same per-lane column ownership (lanes 1..30 of the
// 128-column segment [120 b - 4, 120 b + 124)), rows in ascending order, the same xor tree -- so
// the slots are exactly what a fused launch writing J would have stored.  grid = (nslots), 32
// threads; a.src = J (width x height + the statistics area), fparam[1..4] = ROI.
extern "C" __global__ void __launch_bounds__(32) orion_srad_stats_init(orion_kargs a)
{
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    asm volatile("griddepcontrol.wait;" ::: "memory");
    const SradRoi r = srad_roi(a);
    const int lane = threadIdx.x;
    const int k = blockIdx.x;
    const int g = r.g1 + k / r.nb, b = r.b1 + k % r.nb;
    const int W = a.width, H = a.height;
    const int cx = 120 * b - 4 + 4 * lane;
    const bool own = lane >= 1 && lane <= 30 && cx < W;
    double s = 0.0, s2 = 0.0;
    const int y0 = g * SRADH_RY, y1 = min(y0 + SRADH_RY, H);
    for (int y = y0; y < y1; ++y) {
        if (!own || y < r.r1 || y > r.r2) continue;
        const float4 v = *reinterpret_cast<const float4 *>((const float *)a.src + (size_t)y * (size_t)W + cx);
        srad_roi_acc(s, s2, v, cx, y, r, own);
    }
    srad_roi_store(s, s2, srad_stats_area(a.src, a, 0), g, b, r, lane);
}
