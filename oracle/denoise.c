/*
 * oracle/denoise.c -- TEST INFRASTRUCTURE ONLY (the CPU oracle, part O2).
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
 * reference leg may load this code.  The product path (liborion) never links,
 * includes or calls it, and this file includes nothing from the product.
 *
 * What it computes: the imageDenoising KNN and NLM filters, in double
 * precision, written out as their plain definition, one pixel at a time.
 *
 *   PAPER.md names the benchmark ("imageDenoising program from CUDA
 *   SDK [20]"; Table 2 row P:L733) but never states its math.  The definition
 *   below is SURVEY.md §8(c) O2 (the public CUDA-SDK imageDenoising sample),
 *   adopted as DESIGN.md reading R-O2:
 *
 *   p(u,v) = img[clamp(v,0,H-1)][clamp(u,0,W-1)].rgb   (clamp-to-edge)
 *   c00    = p(x,y)
 *   for i in -R..R (rows), j in -R..R (cols):
 *     KNN:  d = |p(x+j,y+i) - c00|^2                         (sum over r,g,b)
 *     NLM:  d = sum_{n,m in -B..B} |p(x+j+m,y+i+n) - p(x+m,y+n)|^2
 *     w   = exp(-(d*Noise + (i*i+j*j)/A)),   A = (2R+1)^2
 *     acc += w * p(x+j,y+i);  sw += w;  cnt += (w > wthr)
 *   clr = acc / sw
 *   q   = (cnt/A > lthr) ? lerpC : 1 - lerpC
 *   out.rgb = clr + (c00 - clr) * q;     out.a = 0
 *
 * Ambiguous-pixel rule (reading R-AMB): the count
 * is a discontinuous function of w.  A weight with |w - wthr| <= band*wthr is
 * "uncertain" (an fp32 evaluation may land on either side).  The oracle then
 * computes cnt_min / cnt_max; if the lerp branch differs between them the pixel
 * is flagged and BOTH results are returned (out = branch of the double count,
 * alt = the other branch).  Either is a correct fp32 answer.
 *
 * Parity pins (tests/test_oracle_denoise.py): constant image -> identity,
 * Noise -> inf -> identity, flip/transpose equivariance, the closed form of a
 * gray impulse on black, brute force of the double sum by a separate numpy
 * evaluation on tiny inputs.
 */
#include <math.h>
#include <stddef.h>

typedef struct {
    double noise;   /* Noise = 1/h^2 (KNN: 1/0.32^2, NLM: 1/1.45^2)          */
    double lerpc;   /* lerpC = 0.2                                            */
    double wthr;    /* weight threshold (KNN 0.02, NLM 0.10)                  */
    double lthr;    /* lerp threshold on cnt/A (KNN 0.79, NLM 0.10)           */
    double band;    /* relative uncertainty band for the ambiguous-pixel rule */
    int R;          /* window radius (3)                                      */
    int B;          /* patch radius (NLM: 3; KNN: unused)                     */
} oracle_dn_params;

static int clampi(int v, int lo, int hi) { return v < lo ? lo : (v > hi ? hi : v); }

/* p(u,v): image slab holds global rows [row0, row0+nrows) of a W x H image. */
static void sample(const float *img, int W, int H, int row0, int u, int v, double c[3])
{
    int uu = clampi(u, 0, W - 1);
    int vv = clampi(v, 0, H - 1);
    const float *q = img + ((size_t)(vv - row0) * (size_t)W + (size_t)uu) * 4;
    c[0] = q[0]; c[1] = q[1]; c[2] = q[2];
}

static double dist2(const double a[3], const double b[3])
{
    double dx = a[0] - b[0], dy = a[1] - b[1], dz = a[2] - b[2];
    return dx * dx + dy * dy + dz * dz;
}

static double lerp_q(int cnt, int A, const oracle_dn_params *p)
{
    return ((double)cnt / (double)A > p->lthr) ? p->lerpc : 1.0 - p->lerpc;
}

/* One output pixel.  nlm = 0: KNN, 1: NLM. */
static void eval_px(const float *img, int W, int H, int row0, int x, int y,
                    const oracle_dn_params *p, int nlm, double out[3], double alt[3], int *amb)
{
    const int R = p->R, B = p->B;
    const int A = (2 * R + 1) * (2 * R + 1);
    double c00[3];
    sample(img, W, H, row0, x, y, c00);
    double acc[3] = {0.0, 0.0, 0.0}, sw = 0.0;
    int cnt = 0, unsure_in = 0, unsure_out = 0;
    for (int i = -R; i <= R; ++i) {
        for (int j = -R; j <= R; ++j) {
            double cij[3];
            sample(img, W, H, row0, x + j, y + i, cij);
            double d;
            if (!nlm) {
                d = dist2(cij, c00);
            } else {
                d = 0.0;
                for (int n = -B; n <= B; ++n)
                    for (int m = -B; m <= B; ++m) {
                        double a[3], b[3];
                        sample(img, W, H, row0, x + j + m, y + i + n, a);
                        sample(img, W, H, row0, x + m, y + n, b);
                        d += dist2(a, b);
                    }
            }
            double w = exp(-(d * p->noise + (double)(i * i + j * j) / (double)A));
            acc[0] += w * cij[0]; acc[1] += w * cij[1]; acc[2] += w * cij[2];
            sw += w;
            int above = w > p->wthr;
            cnt += above;
            if (fabs(w - p->wthr) <= p->band * p->wthr) {
                if (above) ++unsure_in; else ++unsure_out;
            }
        }
    }
    double clr[3] = {acc[0] / sw, acc[1] / sw, acc[2] / sw};
    double q = lerp_q(cnt, A, p);
    double qmin = lerp_q(cnt - unsure_in, A, p);
    double qmax = lerp_q(cnt + unsure_out, A, p);
    double qalt = (qmin != q) ? qmin : qmax;
    *amb = (qmin != qmax);
    for (int c = 0; c < 3; ++c) {
        out[c] = clr[c] + (c00[c] - clr[c]) * q;
        alt[c] = clr[c] + (c00[c] - clr[c]) * qalt;
    }
}

/*
 * Filter output rows [y_begin, y_end) (global) of a W x H image.
 * img: float32 RGBA slab of global rows [row0, row0+nrows) -- must contain every
 *      row the window (and patch) reaches after clamping.
 * out, alt: double rgb, (y_end-y_begin) x W x 3.  amb: int (y_end-y_begin) x W.
 * Returns the number of ambiguous pixels.
 */
long oracle_denoise_rows(const float *img, int W, int H, int row0, int nrows,
                         int y_begin, int y_end, const oracle_dn_params *p, int nlm,
                         double *out, double *alt, int *amb)
{
    (void)nrows;
    long n_amb = 0;
    for (int y = y_begin; y < y_end; ++y)
        for (int x = 0; x < W; ++x) {
            size_t o = (size_t)(y - y_begin) * (size_t)W + (size_t)x;
            eval_px(img, W, H, row0, x, y, p, nlm, out + 3 * o, alt + 3 * o, amb + o);
            n_amb += amb[o];
        }
    return n_amb;
}

/* Filter an explicit list of n pixels (xs[k], ys[k]); same outputs per pixel. */
long oracle_denoise_points(const float *img, int W, int H, int row0, int nrows,
                           const int *xs, const int *ys, int n, const oracle_dn_params *p, int nlm,
                           double *out, double *alt, int *amb)
{
    (void)nrows;
    long n_amb = 0;
    for (int k = 0; k < n; ++k) {
        eval_px(img, W, H, row0, xs[k], ys[k], p, nlm, out + 3 * (size_t)k, alt + 3 * (size_t)k, amb + k);
        n_amb += amb[k];
    }
    return n_amb;
}
