/*
 * oracle/stencil.c -- TEST INFRASTRUCTURE ONLY (the CPU oracle, part O3).
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
 * reference leg may load this code; the product never links or calls it.
 *
 * What it computes: the Rodinia-style 2-D thermal stencil ("hotspot", PAPER.md
 * Table 2 row P:L731, Rodinia [6] P:L1147).  The paper gives no formula; the
 * update below is SURVEY.md §8(c) O3 (Rodinia hotspot), reading R-O3:
 *
 *   T'[y][x] = T + sdc * ( P + (T[S] + T[N] - 2T)*ry + (T[E] + T[W] - 2T)*rx + (amb - T)*rz )
 *
 * with clamp-to-edge neighbours (zero-flux boundary) and the fixed-cell-size
 * constants of reading R-A15 (sdc = step/Cap, rx = 1/Rx, ry = 1/Ry, rz = 1/Rz).
 * One call = `steps` explicit steps (ping-pong buffers).
 *
 * Two forms:
 *   oracle_hotspot_f64 -- the definition in double precision;
 *   oracle_hotspot_f32 -- the same definition evaluated in fp32, every operation
 *     rounded once, in the order written above, with the products that feed a sum
 *     fused (reading R-HS-FP; explicit fmaf, the file is compiled with
 *     -ffp-contract=off so nothing else is contracted):
 *       a = fma(T, -2, S + N);   b = fma(T, -2, E + W);   d = amb - T;
 *       acc = fma(rz, d, fma(rx, b, fma(ry, a, P)));      T' = fma(sdc, acc, T)
 *
 * Pins (tests/test_oracle_stencil.py): uniform T = amb, P = 0 is a fixed point;
 * the discrete Neumann cosine modes are eigenvectors with a closed-form
 * eigenvalue (checked after many steps); heat conservation with rz = 0, P = 0;
 * the maximum principle; f32 form within the fp32 error bound of f64.
 */
#include <math.h>
#include <stddef.h>
#include <stdlib.h>
#include <string.h>

typedef struct { double sdc, rx, ry, rz, amb; } oracle_hs_params;

static int clampi(int v, int lo, int hi) { return v < lo ? lo : (v > hi ? hi : v); }

int oracle_hotspot_f64(const double *t0, const double *power, int W, int H, int steps,
                       const oracle_hs_params *p, double *out)
{
    size_t n = (size_t)W * (size_t)H;
    double *a = (double *)malloc(n * sizeof(double));
    double *b = (double *)malloc(n * sizeof(double));
    if (!a || !b) { free(a); free(b); return -1; }
    for (size_t k = 0; k < n; ++k) a[k] = t0[k];
    for (int s = 0; s < steps; ++s) {
        for (int y = 0; y < H; ++y)
            for (int x = 0; x < W; ++x) {
                double T = a[(size_t)y * W + x];
                double N = a[(size_t)clampi(y - 1, 0, H - 1) * W + x];
                double S = a[(size_t)clampi(y + 1, 0, H - 1) * W + x];
                double Wv = a[(size_t)y * W + clampi(x - 1, 0, W - 1)];
                double E = a[(size_t)y * W + clampi(x + 1, 0, W - 1)];
                double P = power[(size_t)y * W + x];
                b[(size_t)y * W + x] = T + p->sdc * (P + (S + N - 2.0 * T) * p->ry
                                                       + (E + Wv - 2.0 * T) * p->rx
                                                       + (p->amb - T) * p->rz);
            }
        double *t = a; a = b; b = t;
    }
    memcpy(out, a, n * sizeof(double));
    free(a); free(b);
    return 0;
}

int oracle_hotspot_f32(const float *t0, const float *power, int W, int H, int steps,
                       const oracle_hs_params *p, float *out)
{
    size_t n = (size_t)W * (size_t)H;
    float *a = (float *)malloc(n * sizeof(float));
    float *b = (float *)malloc(n * sizeof(float));
    if (!a || !b) { free(a); free(b); return -1; }
    const float sdc = (float)p->sdc, rx = (float)p->rx, ry = (float)p->ry, rz = (float)p->rz,
                amb = (float)p->amb;
    memcpy(a, t0, n * sizeof(float));
    for (int s = 0; s < steps; ++s) {
        for (int y = 0; y < H; ++y)
            for (int x = 0; x < W; ++x) {
                float T = a[(size_t)y * W + x];
                float N = a[(size_t)clampi(y - 1, 0, H - 1) * W + x];
                float S = a[(size_t)clampi(y + 1, 0, H - 1) * W + x];
                float Wv = a[(size_t)y * W + clampi(x - 1, 0, W - 1)];
                float E = a[(size_t)y * W + clampi(x + 1, 0, W - 1)];
                float P = power[(size_t)y * W + x];
                float av = fmaf(T, -2.0f, S + N);
                float bv = fmaf(T, -2.0f, E + Wv);
                float dv = amb - T;
                float acc = fmaf(rz, dv, fmaf(rx, bv, fmaf(ry, av, P)));
                b[(size_t)y * W + x] = fmaf(sdc, acc, T);
            }
        float *t = a; a = b; b = t;
    }
    memcpy(out, a, n * sizeof(float));
    free(a); free(b);
    return 0;
}
