/*
 * oracle/srad.c -- TEST INFRASTRUCTURE ONLY (the CPU oracle, part O5).
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference
 * leg may load this code; the product never links or calls it.
 *
 * What it computes: SRAD, speckle-reducing anisotropic diffusion (Table 2 row
 * P:L739 "srad [6] Imaging app", Fig. 10 P:L657-L693 -- the paper's downward-tuning
 * example).  The paper gives no formula; the update below is Rodinia's srad_v2 (ref [6],
 * P:L1147), adopted as DESIGN.md reading R-SRAD.  One iteration:
 *
 *   ROI statistics over rows [r1, r2] x cols [c1, c2] (inclusive):
 *     mean = sum/n;  var = sum2/n - mean^2;  q0sqr = var / mean^2
 *   per cell (clamp-to-edge neighbours N, S, W, E of J):
 *     dN = J[N]-J, dS = J[S]-J, dW = J[W]-J, dE = J[E]-J
 *     G2 = (dN^2 + dS^2 + dW^2 + dE^2) / J^2
 *     L  = (dN + dS + dW + dE) / J
 *     num = 0.5*G2 - (1/16)*L^2;  den = 1 + 0.25*L;  qsqr = num / den^2
 *     den = (qsqr - q0sqr) / (q0sqr * (1 + q0sqr));  c = 1 / (1 + den), clamped to [0, 1]
 *   per cell:
 *     D = c*dN + c[S]*dS + c*dW + c[E]*dE;   J' = J + 0.25*lambda*D
 *
 * Pins (tests/test_oracle_srad.py): total intensity is conserved (the update is in
 * divergence form with zero-flux borders); the maximum principle for lambda <= 1;
 * lambda = 0 is the identity; flip equivariance where the stencil is symmetric (a
 * mirrored image with a mirrored ROI); the ROI statistics against numpy.
 */
#include <math.h>
#include <stdlib.h>
#include <string.h>

static int clampi(int v, int lo, int hi) { return v < lo ? lo : (v > hi ? hi : v); }

int oracle_srad_f64(const double *j0, int W, int H, int iters, double lambda, int r1, int r2, int c1, int c2,
                    double *out, double *q0_out)
{
    size_t n = (size_t)W * (size_t)H;
    double *J = (double *)malloc(n * sizeof(double));
    double *C = (double *)malloc(n * sizeof(double));
    if (!J || !C) { free(J); free(C); return -1; }
    memcpy(J, j0, n * sizeof(double));
    for (int it = 0; it < iters; ++it) {
        double sum = 0.0, sum2 = 0.0;
        for (int i = r1; i <= r2; ++i)
            for (int j = c1; j <= c2; ++j) {
                double t = J[(size_t)i * W + j];
                sum += t;
                sum2 += t * t;
            }
        double size = (double)(r2 - r1 + 1) * (double)(c2 - c1 + 1);
        double mean = sum / size;
        double var = sum2 / size - mean * mean;
        double q0sqr = var / (mean * mean);
        if (q0_out) q0_out[it] = q0sqr;
        for (int i = 0; i < H; ++i)
            for (int j = 0; j < W; ++j) {
                double Jc = J[(size_t)i * W + j];
                double dN = J[(size_t)clampi(i - 1, 0, H - 1) * W + j] - Jc;
                double dS = J[(size_t)clampi(i + 1, 0, H - 1) * W + j] - Jc;
                double dW = J[(size_t)i * W + clampi(j - 1, 0, W - 1)] - Jc;
                double dE = J[(size_t)i * W + clampi(j + 1, 0, W - 1)] - Jc;
                double G2 = (dN * dN + dS * dS + dW * dW + dE * dE) / (Jc * Jc);
                double L = (dN + dS + dW + dE) / Jc;
                double num = 0.5 * G2 - (1.0 / 16.0) * (L * L);
                double den = 1.0 + 0.25 * L;
                double qsqr = num / (den * den);
                den = (qsqr - q0sqr) / (q0sqr * (1.0 + q0sqr));
                double c = 1.0 / (1.0 + den);
                C[(size_t)i * W + j] = c < 0.0 ? 0.0 : (c > 1.0 ? 1.0 : c);
            }
        double *Jn = (double *)malloc(n * sizeof(double));
        if (!Jn) { free(J); free(C); return -1; }
        for (int i = 0; i < H; ++i)
            for (int j = 0; j < W; ++j) {
                double Jc = J[(size_t)i * W + j];
                int iS = clampi(i + 1, 0, H - 1), jE = clampi(j + 1, 0, W - 1);
                double dN = J[(size_t)clampi(i - 1, 0, H - 1) * W + j] - Jc;
                double dS = J[(size_t)iS * W + j] - Jc;
                double dW = J[(size_t)i * W + clampi(j - 1, 0, W - 1)] - Jc;
                double dE = J[(size_t)i * W + jE] - Jc;
                double cN = C[(size_t)i * W + j], cS = C[(size_t)iS * W + j];
                double cW = cN, cE = C[(size_t)i * W + jE];
                double D = cN * dN + cS * dS + cW * dW + cE * dE;
                Jn[(size_t)i * W + j] = Jc + 0.25 * lambda * D;
            }
        free(J);
        J = Jn;
    }
    memcpy(out, J, n * sizeof(double));
    free(J);
    free(C);
    return 0;
}
