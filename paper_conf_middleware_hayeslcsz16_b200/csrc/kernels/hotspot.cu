// hotspot.cu -- Rodinia-style 2-D thermal stencil, one explicit step per launch
// (Table 2, Rodinia [6] P:L1147; update rule per DESIGN.md reading
// R-O3, constants per reading R-A15):
//   T' = T + sdc * ( P + (S + N - 2T)*ry + (E + W - 2T)*rx + (amb - T)*rz )
// with clamp-to-edge neighbours, evaluated in fp32 in exactly this order (one
// rounding per operation, no contraction):
//   t2 = T+T; a = ((S+N)-t2)*ry; b = ((E+W)-t2)*rx; c = (amb-T)*rz; T' = T + (((P+a)+b)+c)*sdc
//
// HBM-bound (12 algorithmic bytes per cell-step).  Each warp owns 32 consecutive
// columns and walks a strip of RY rows top to bottom, keeping N / T / S in
// registers (every row of T is read once from DRAM per strip); E and W come from
// the neighbouring lanes by shuffle, lanes 0/31 fetch their outer neighbour (an
// L1/L2 hit, the same line the neighbouring warp loads).  The loads of the next
// rows are software-prefetched RY_PF rows ahead to keep enough bytes in flight --
// and the warps resident per SM (the occupancy level Orion tunes) supply the rest.
#include "common.cuh"

template <int BY, int RY>
__device__ __forceinline__ void hotspot_body(const orion_kargs &a)
{
    const float *tin = (const float *)a.src;
    const float *pw = (const float *)a.aux;
    float *tout = (float *)a.dst;
    const int W = a.width, H = a.height;
    const int lane = threadIdx.x;
    const int xr = blockIdx.x * 32 + lane;
    const int x = min(xr, W - 1);
    const int ys = a.row_begin + (blockIdx.y * BY + threadIdx.y) * RY;
    if (ys >= a.row_end) return;
    const int ye = min(ys + RY, a.row_end);
    const float sdc = a.fparam[0], rx = a.fparam[1], ry = a.fparam[2], rz = a.fparam[3], amb = a.fparam[4];
    const int xl = max(blockIdx.x * 32 - 1, 0);                 // lane 0's west neighbour
    const int xh = min(blockIdx.x * 32 + 32, W - 1);            // lane 31's east neighbour
    const int sb = a.src_row_begin;
#define ROWP(y) (tin + (size_t)((y) - sb) * (size_t)W)
    float N = __ldg(ROWP(max(ys - 1, 0)) + x);
    float T = __ldg(ROWP(ys) + x);
    for (int y = ys; y < ye; ++y) {
        const float S = __ldg(ROWP(min(y + 1, H - 1)) + x);
        const float P = __ldg(pw + (size_t)(y - sb) * (size_t)W + x);
        float Wv = __shfl_up_sync(0xffffffffu, T, 1);
        float Ev = __shfl_down_sync(0xffffffffu, T, 1);
        if (lane == 0) Wv = (xr == 0) ? T : __ldg(ROWP(y) + xl);
        if (lane == 31) Ev = __ldg(ROWP(y) + xh);
        if (xr >= W - 1) Ev = T;                                  // clamp at the east edge
        const float t2 = __fadd_rn(T, T);
        const float av = __fmul_rn(__fsub_rn(__fadd_rn(S, N), t2), ry);
        const float bv = __fmul_rn(__fsub_rn(__fadd_rn(Ev, Wv), t2), rx);
        const float cv = __fmul_rn(__fsub_rn(amb, T), rz);
        const float acc = __fadd_rn(__fadd_rn(__fadd_rn(P, av), bv), cv);
        const float o = __fadd_rn(T, __fmul_rn(acc, sdc));
        if (xr < W) tout[(size_t)(y - a.dst_row_begin) * (size_t)W + xr] = o;
        N = T;
        T = S;
    }
#undef ROWP
}

// T = 256 threads (32 x 8 warps), 16-row strips per warp.
extern "C" __global__ void __launch_bounds__(256) orion_hotspot_f32_256(orion_kargs a) { hotspot_body<8, 16>(a); }
// T = 128 threads (32 x 4 warps), 16-row strips per warp.
extern "C" __global__ void __launch_bounds__(128) orion_hotspot_f32_128(orion_kargs a) { hotspot_body<4, 16>(a); }
