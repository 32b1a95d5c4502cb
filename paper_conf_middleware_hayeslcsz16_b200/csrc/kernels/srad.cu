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
// Update kernel: CTA = 32 x 8 threads, output tile 32 x 32 cells (4 rows per thread).
// The J tile with a 1-cell halo (+1 extra row / column south / east for the neighbours'
// coefficients) is staged in shared memory; the coefficients c of the tile plus one row
// south and one column east are computed once into shared memory (the two-kernel
// Rodinia form writes c and four derivative arrays to DRAM instead); then J' is formed.
// HBM: 8 algorithmic bytes per cell-iteration (read J, write J').
#include "common.cuh"

namespace {
constexpr int SX = 32, SY = 8, RY = 4;        // threads, rows per thread
constexpr int TW = SX, TH = SY * RY;          // output tile 32 x 32
constexpr int JW = TW + 3, JH = TH + 3;       // J tile: x0-1 .. x0+TW+1, y0-1 .. y0+TH+1
constexpr int CW = TW + 1, CH = TH + 1;       // c tile: x0 .. x0+TW, y0 .. y0+TH
}  // namespace

extern "C" __global__ void __launch_bounds__(256) orion_srad_f32_256(orion_kargs a)
{
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
    const float q0 = *(const float *)a.aux;
    const float lam4 = __fmul_rn(0.25f, a.fparam[0]);
    const float iqden = __frcp_rn(__fmul_rn(q0, __fadd_rn(1.0f, q0)));
    __syncthreads();
    // coefficient tile: cell (y0+cy, x0+cx), cy in [0, CH), cx in [0, CW).  The cell at
    // global (gy, gx) with gy >= H or gx >= W is a clamped copy: its coefficient is the
    // edge cell's, which the clamped J values reproduce (all its neighbours clamp alike).
    for (int idx = tid; idx < CW * CH; idx += SX * SY) {
        const int cy = idx / CW, cx = idx - cy * CW;
        const int gy = y0 + cy, gx = x0 + cx;
        // tile coordinates of (gy, gx) and its clamped neighbours
        const int ty = min(gy, H - 1) - (y0 - 1), tx = min(gx, W - 1) - (x0 - 1);
        const int tn = max(min(gy, H - 1) - 1, 0) - (y0 - 1), ts = min(min(gy, H - 1) + 1, H - 1) - (y0 - 1);
        const int tw = max(min(gx, W - 1) - 1, 0) - (x0 - 1), te = min(min(gx, W - 1) + 1, W - 1) - (x0 - 1);
        const float Jc = js[ty * JW + tx];
        const float dN = __fsub_rn(js[tn * JW + tx], Jc), dS = __fsub_rn(js[ts * JW + tx], Jc);
        const float dW = __fsub_rn(js[ty * JW + tw], Jc), dE = __fsub_rn(js[ty * JW + te], Jc);
        const float g2n = __fadd_rn(__fadd_rn(__fadd_rn(__fmul_rn(dN, dN), __fmul_rn(dS, dS)), __fmul_rn(dW, dW)),
                                    __fmul_rn(dE, dE));
        // one IEEE reciprocal of J serves G2 = sum d^2 / J^2 and L = sum d / J; the
        // (qsqr - q0sqr) / (q0sqr (1 + q0sqr)) division uses the launch-uniform reciprocal
        const float ij = __frcp_rn(Jc);
        const float G2 = __fmul_rn(__fmul_rn(g2n, ij), ij);
        const float L = __fmul_rn(__fadd_rn(__fadd_rn(__fadd_rn(dN, dS), dW), dE), ij);
        const float num = __fsub_rn(__fmul_rn(0.5f, G2), __fmul_rn(0.0625f, __fmul_rn(L, L)));
        const float den = __fadd_rn(1.0f, __fmul_rn(0.25f, L));
        const float qsqr = __fdiv_rn(num, __fmul_rn(den, den));
        const float dd = __fmul_rn(__fsub_rn(qsqr, q0), iqden);
        const float c = __frcp_rn(__fadd_rn(1.0f, dd));
        cs[idx] = fminf(fmaxf(c, 0.0f), 1.0f);
    }
    __syncthreads();
    const int cx = threadIdx.x, gx = x0 + cx;
    if (gx >= W) return;
#pragma unroll
    for (int r = 0; r < RY; ++r) {
        const int cy = threadIdx.y * RY + r, gy = y0 + cy;
        if (gy >= a.row_end) return;
        const int ty = gy - (y0 - 1), tx = gx - (x0 - 1);
        const int tn = max(gy - 1, 0) - (y0 - 1), ts = min(gy + 1, H - 1) - (y0 - 1);
        const int tw = max(gx - 1, 0) - (x0 - 1), te = min(gx + 1, W - 1) - (x0 - 1);
        const float Jc = js[ty * JW + tx];
        const float dN = __fsub_rn(js[tn * JW + tx], Jc), dS = __fsub_rn(js[ts * JW + tx], Jc);
        const float dW = __fsub_rn(js[ty * JW + tw], Jc), dE = __fsub_rn(js[ty * JW + te], Jc);
        const float cC = cs[cy * CW + cx];
        const float cS = cs[(min(gy + 1, H - 1) - y0) * CW + cx];
        const float cE = cs[cy * CW + (min(gx + 1, W - 1) - x0)];
        const float D = __fadd_rn(__fadd_rn(__fadd_rn(__fmul_rn(cC, dN), __fmul_rn(cS, dS)), __fmul_rn(cC, dW)),
                                  __fmul_rn(cE, dE));
        ((float *)a.dst)[(size_t)(gy - a.dst_row_begin) * (size_t)W + gx] = __fadd_rn(Jc, __fmul_rn(lam4, D));
    }
}

// ROI statistics: one CTA of 1024 threads; thread t sums elements t, t+1024, ... of the
// row-major ROI in double, then a fixed-shape tree in shared memory -- deterministic, so
// every occupancy variant of the update kernel sees the same q0sqr.
extern "C" __global__ void __launch_bounds__(1024) orion_srad_stats(const float *J, int W, int r1, int r2, int c1,
                                                                     int c2, float *q0)
{
    __shared__ double s1[1024], s2[1024];
    const int t = threadIdx.x;
    const int rw = c2 - c1 + 1, n = (r2 - r1 + 1) * rw;
    double a = 0.0, b = 0.0;
    for (int e = t; e < n; e += 1024) {
        const int i = r1 + e / rw, j = c1 + e % rw;
        const double v = J[(size_t)i * (size_t)W + j];
        a += v;
        b += v * v;
    }
    s1[t] = a;
    s2[t] = b;
    __syncthreads();
    for (int s = 512; s > 0; s >>= 1) {
        if (t < s) {
            s1[t] += s1[t + s];
            s2[t] += s2[t + s];
        }
        __syncthreads();
    }
    if (t == 0) {
        const double mean = s1[0] / n;
        const double var = s2[0] / n - mean * mean;
        *q0 = (float)(var / (mean * mean));
    }
}

// ---- register-sliding variant ------------------------------------------------------------
// Same arithmetic, no shared memory: lane l of a warp owns column x0 + l (x0 = 31 * block
// column; lanes 0..30 write, lane 31 only supplies the coefficient its west neighbour needs
// as c_E) and walks a strip of RY rows keeping J rows y-1 .. y+2 and the coefficients of rows
// y, y+1 in registers.  E / W neighbours come by shuffle; lanes 0 / 31 load the column just
// outside the warp.  One coefficient per cell, one coalesced 128-byte row load per step.
namespace {
struct JRow {
    float c, w, e;   // J at the lane's column and at its west / east neighbours
};
}  // namespace

template <int BY, int RY>
__device__ __forceinline__ void srad2_body(const orion_kargs &a)
{
    const float *J = (const float *)a.src;
    float *Jo = (float *)a.dst;
    const int W = a.width, H = a.height;
    const int lane = threadIdx.x;
    const int x0 = blockIdx.x * 31;
    const int xr = x0 + lane;
    const int x = min(xr, W - 1);
    const int ys = a.row_begin + (blockIdx.y * BY + threadIdx.y) * RY;
    if (ys >= a.row_end) return;
    const int ye = min(ys + RY, a.row_end);
    const size_t sb = (size_t)a.src_row_begin;
    const float q0 = *(const float *)a.aux;
    const float lam4 = __fmul_rn(0.25f, a.fparam[0]);
    const float iqden = __frcp_rn(__fmul_rn(q0, __fadd_rn(1.0f, q0)));
    const int xw = clampi(x0 - 1, 0, W - 1), xe = clampi(x0 + 32, 0, W - 1);

    auto load = [&](int y) {
        const float *row = J + ((size_t)y - sb) * (size_t)W;
        JRow r;
        r.c = __ldg(row + x);
        r.w = __shfl_up_sync(0xffffffffu, r.c, 1);
        r.e = __shfl_down_sync(0xffffffffu, r.c, 1);
        if (lane == 0) r.w = __ldg(row + xw);
        if (lane == 31) r.e = __ldg(row + xe);
        if (xr == 0) r.w = r.c;                       // clamp at the west edge
        if (xr >= W - 1) r.e = r.c;                   // clamp at the east edge
        return r;
    };
    // diffusion coefficient of the cell (row of T, north row N, south row S)
    auto coeff = [&](const JRow &T, float Nc, float Sc) {
        const float Jc = T.c;
        const float dN = __fsub_rn(Nc, Jc), dS = __fsub_rn(Sc, Jc);
        const float dW = __fsub_rn(T.w, Jc), dE = __fsub_rn(T.e, Jc);
        const float g2n = __fadd_rn(__fadd_rn(__fadd_rn(__fmul_rn(dN, dN), __fmul_rn(dS, dS)), __fmul_rn(dW, dW)),
                                    __fmul_rn(dE, dE));
        const float ij = __frcp_rn(Jc);
        const float G2 = __fmul_rn(__fmul_rn(g2n, ij), ij);
        const float L = __fmul_rn(__fadd_rn(__fadd_rn(__fadd_rn(dN, dS), dW), dE), ij);
        const float num = __fsub_rn(__fmul_rn(0.5f, G2), __fmul_rn(0.0625f, __fmul_rn(L, L)));
        const float den = __fadd_rn(1.0f, __fmul_rn(0.25f, L));
        const float qsqr = __fdiv_rn(num, __fmul_rn(den, den));
        const float dd = __fmul_rn(__fsub_rn(qsqr, q0), iqden);
        return fminf(fmaxf(__frcp_rn(__fadd_rn(1.0f, dd)), 0.0f), 1.0f);
    };
    JRow jm = load(max(ys - 1, 0)), j0 = load(ys), j1 = load(min(ys + 1, H - 1));
    float c0 = coeff(j0, jm.c, j1.c);
    for (int y = ys; y < ye; ++y) {
        const JRow j2 = load(min(y + 2, H - 1));
        const float c1 = (y + 1 <= H - 1) ? coeff(j1, j0.c, j2.c) : c0;   // c of row clamp(y+1)
        float cE = __shfl_down_sync(0xffffffffu, c0, 1);
        if (xr >= W - 1) cE = c0;
        const float Jc = j0.c;
        const float dN = __fsub_rn(jm.c, Jc), dS = __fsub_rn(j1.c, Jc);
        const float dW = __fsub_rn(j0.w, Jc), dE = __fsub_rn(j0.e, Jc);
        const float D = __fadd_rn(__fadd_rn(__fadd_rn(__fmul_rn(c0, dN), __fmul_rn(c1, dS)), __fmul_rn(c0, dW)),
                                  __fmul_rn(cE, dE));
        if (lane < 31 && xr < W)
            Jo[((size_t)y - (size_t)a.dst_row_begin) * (size_t)W + xr] = __fadd_rn(Jc, __fmul_rn(lam4, D));
        jm = j0;
        j0 = j1;
        j1 = j2;
        c0 = c1;
    }
}

// T = 256 threads (32 x 8 warps): 31 output columns x 8 strips of 16 rows per CTA.
extern "C" __global__ void __launch_bounds__(256) orion_srad2_f32_256(orion_kargs a) { srad2_body<8, 16>(a); }
