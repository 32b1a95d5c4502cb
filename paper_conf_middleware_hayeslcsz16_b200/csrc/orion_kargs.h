/* orion_kargs.h -- the by-value parameter block every Orion kernel receives.
 * Shared by the host launcher (g++) and the kernels (nvcc -> PTX); product-internal.
 * Layout must stay identical on both sides (plain 4/8-byte fields, no padding surprises). */
#ifndef ORION_KARGS_H
#define ORION_KARGS_H

typedef struct {
    const void *src;      /* rows [src_row_begin, src_row_end) of a width-wide image, pitch = width */
    void *dst;            /* rows [dst_row_begin, ...), pitch = width                               */
    const void *aux;      /* stencil power map (same rows as src); NULL for the denoisers            */
    int width, height;    /* global image size                                                      */
    int row_begin, row_end;          /* output rows computed by this launch (global)                */
    int src_row_begin, src_row_end;  /* rows held by src (global)                                   */
    int dst_row_begin;               /* global row of dst's first row                               */
    int iparam0;                     /* denoise: lerp count threshold (cnt >= iparam0 -> lerpC)     */
    float fparam[8];                 /* denoise: -Noise*log2e, lerpC, wthr ; stencil: sdc,rx,ry,rz,amb */
    unsigned *probe;                 /* NULL in every real launch.  Non-NULL: residency probe only --
                                        the CTA records how many CTAs share its SM and exits
                                        (orion_probe in kernels/common.cuh)                        */
    void *fan[8];                    /* denoisers: extra full-image outputs (global row y at y*width), */
    int nfan;                        /* e.g. every rank's gather buffer over NVLink peer memory        */
    int nowait;                      /* 1: no griddepcontrol.wait (ORION_ARGS_INDEPENDENT, or a chained
                                        launch whose predecessor is the same chain's previous launch) */
    int dep_late;                    /* 1: the kernel issues griddepcontrol.launch_dependents itself,
                                        later than at entry (chained srad_f32hs: after its slot reads) */
    unsigned *chain;                 /* orion_chain tile flags (gridDim.y x gridDim.x); NULL: none     */
    unsigned chain_epoch;            /* this launch's epoch; it waits for epoch-1 on the tiles it reads */
    int batch;                       /* frames of a batched denoiser launch (gridDim.z); 1 otherwise    */
} orion_kargs;

#endif
