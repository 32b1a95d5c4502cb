// hotspot.cu -- Rodinia-style 2-D thermal stencil, one explicit step per launch
// (Table 2, Rodinia [6] P:L1147; update rule per DESIGN.md reading
// R-O3, constants per reading R-A15):
//   T' = T + sdc * ( P + (S + N - 2T)*ry + (E + W - 2T)*rx + (amb - T)*rz )
// with clamp-to-edge neighbours, evaluated in fp32 in exactly this order (one
// rounding per operation, no contraction):
//   t2 = T+T; a = ((S+N)-t2)*ry; b = ((E+W)-t2)*rx; c = (amb-T)*rz; T' = T + (((P+a)+b)+c)*sdc
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
    const float t2 = __fadd_rn(T, T);
    const float av = __fmul_rn(__fsub_rn(__fadd_rn(S, N), t2), c[2]);
    const float bv = __fmul_rn(__fsub_rn(__fadd_rn(E, Wv), t2), c[1]);
    const float cv = __fmul_rn(__fsub_rn(c[4], T), c[3]);
    const float acc = __fadd_rn(__fadd_rn(__fadd_rn(P, av), bv), cv);
    return __fadd_rn(T, __fmul_rn(acc, c[0]));
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
            float4 o;
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

// ---- two explicit steps per launch (temporal blocking) -------------------------------------
// T2 = step(step(T0)) with the intermediate T1 kept in registers: per 2 cell-steps the kernel
// reads T0 and P once and writes T2 once (12 B instead of 24 B of DRAM traffic).  Each warp
// walks a strip of rows computing T1 one row ahead of T2; E / W neighbours come by shuffle,
// and lanes 0 / 31 also compute the T1 cell just outside the warp's 128 columns (the halo
// the outer T2 cells need), from predicated scalar loads.  Every cell value is produced by
// the same hs_cell() as the one-step kernel, with the same clamp-to-edge neighbours, so two
// one-step launches and one two-step launch give identical bits.  Rows must be 16-byte
// aligned (width % 4 == 0; the launcher rejects other widths for this kernel).
struct Row4 {
    float4 v;      // own columns cx .. cx+3
    float xw, xe;  // T at the warp's outer neighbours: cx0-1 (lane 0), cx0+128 (lane 31)
    float xo;      // T one further out: cx0-2 (lane 0), cx0+129 (lane 31)
};

template <int BY, int RY>
__device__ __forceinline__ void hotspot2_body(const orion_kargs &a)
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
    const int cx = (blockIdx.x * 32 + lane) * 4;
    const int cxl = min(cx, W - 4);
    const int base = blockIdx.x * 128;
    const bool west_edge = base == 0, east_edge = base + 128 >= W;
    const bool edge_lane = (lane == 0 && !west_edge) || (lane == 31 && !east_edge);
    // the extra column of an edge lane and the one beyond it (valid only on edge lanes)
    const int xx = lane == 0 ? base - 1 : base + 128;
    const int xo = lane == 0 ? base - 2 : base + 129;

    auto load = [&](int y) {
        Row4 r;
        const float *row = tin + ((size_t)y - sb) * (size_t)W;
        r.v = __ldg(reinterpret_cast<const float4 *>(row + cxl));
        r.xw = r.xe = r.xo = 0.0f;
        if (edge_lane) {
            r.xw = r.xe = __ldg(row + xx);
            r.xo = __ldg(row + clampi(xo, 0, W - 1));
        }
        return r;
    };
    // one explicit step of the lane's 4 cells and (edge lanes) of its extra cell
    auto step = [&](const Row4 &N, const Row4 &T, const Row4 &S, float4 P, float Pe, Row4 &out) {
        float Wv = __shfl_up_sync(0xffffffffu, T.v.w, 1);
        float Ev = __shfl_down_sync(0xffffffffu, T.v.x, 1);
        if (lane == 0) Wv = west_edge ? T.v.x : T.xw;
        if (lane == 31) Ev = east_edge ? T.v.w : T.xe;
        if (cx + 4 >= W) Ev = T.v.w;
        if (cx == 0) Wv = T.v.x;
        out.v.x = hs_cell(T.v.x, N.v.x, S.v.x, T.v.y, Wv, P.x, c);
        out.v.y = hs_cell(T.v.y, N.v.y, S.v.y, T.v.z, T.v.x, P.y, c);
        out.v.z = hs_cell(T.v.z, N.v.z, S.v.z, T.v.w, T.v.y, P.z, c);
        out.v.w = hs_cell(T.v.w, N.v.w, S.v.w, Ev, T.v.z, P.w, c);
        // extra cell: lane 0 at base-1 (E = own column base, W = base-2 clamped);
        // lane 31 at base+128 (W = own column base+127, E = base+129 clamped)
        const float te = T.xw;
        const float ee = lane == 0 ? T.v.x : (xo > W - 1 ? te : T.xo);
        const float we = lane == 0 ? (xo < 0 ? te : T.xo) : T.v.w;
        out.xw = out.xe = hs_cell(te, N.xw, S.xw, ee, we, Pe, c);
        out.xo = 0.0f;
    };
    auto prow = [&](int y, float4 &P, float &Pe) {
        const float *row = pw + ((size_t)y - sb) * (size_t)W;
        P = __ldg(reinterpret_cast<const float4 *>(row + cxl));
        Pe = edge_lane ? __ldg(row + xx) : 0.0f;
    };

    const int r_lo = max(ys - 1, 0), r_hi = min(ye, H - 1);
    Row4 t0p = load(max(r_lo - 1, 0)), t0c = load(r_lo);
    Row4 ua, ub, uc;                 // T1 rows r-2, r-1, r
    float4 Pb = make_float4(0.f, 0.f, 0.f, 0.f);
    float Peb = 0.0f;                // P of row r-1 (what T2(r-1) needs)
    bool have_b = false, have_a = false;
    float *orow_base = tout + (size_t)cx;
    for (int r = r_lo; r <= r_hi; ++r) {
        const Row4 t0n = load(min(r + 1, H - 1));
        float4 P;
        float Pe;
        prow(r, P, Pe);
        step(t0p, t0c, t0n, P, Pe, uc);     // T1(r)
        t0p = t0c;
        t0c = t0n;
        const int y = r - 1;                 // T2(y) needs T1(clamp(y-1)), T1(y), T1(r)
        if (have_b && y >= ys && y < ye) {
            Row4 o;
            step(have_a ? ua : ub, ub, uc, Pb, Peb, o);
            if (cx < W) *reinterpret_cast<float4 *>(orow_base + ((size_t)y - db) * (size_t)W) = o.v;
        }
        ua = ub;
        have_a = have_b && (y >= 0);
        ub = uc;
        have_b = true;
        Pb = P;
        Peb = Pe;
    }
    // the bottom row of the image: its south T1 neighbour is itself
    if (ye == H && H - 1 >= ys) {
        Row4 o;
        step(have_a ? ua : ub, ub, ub, Pb, Peb, o);
        if (cx < W) *reinterpret_cast<float4 *>(orow_base + ((size_t)(H - 1) - db) * (size_t)W) = o.v;
    }
}

// T = 256 threads (32 x 8 warps): 128 columns x 8 strips of 16 rows per CTA; 2 steps per launch.
extern "C" __global__ void __launch_bounds__(256) orion_hotspot2_f32_256(orion_kargs a) { ORION_PROBE(a); hotspot2_body<8, 16>(a); }
