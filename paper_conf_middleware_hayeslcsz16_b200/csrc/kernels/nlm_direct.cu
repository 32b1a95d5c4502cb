// nlm_direct.cu -- imageDenoising NLM filter, direct patch-distance form
// (Table 2; math per DESIGN.md reading R-O2).
//
// Per pixel and per window offset (i, j): the 7x7-patch SSD
//   d = sum_{n,m} |p(x+j+m, y+i+n) - p(x+m, y+n)|^2
// then the KNN-style weight / count / lerp.  2401 patch terms per pixel.
//
// Two kernels share this file:
//  * orion_nlm_direct_f4_*: the shifted and the centre patch are both read from the
//    shared-memory tile (low register use, LDS-bound);
//  * orion_nlm_regheavy_f4_*: the SDK-style "register-heavy" variant of config C4 --
//    the centre patch (49 x rgb = 147 values) is held in registers across all 49
//    offsets and the patch loops are fully unrolled; ptxas naturally needs 255
//    registers plus spill, so register caps trade spill traffic for occupancy
//    ("avoid excessive spilling", Table 2 Reg column).
// Tile: BX x BY pixels (1 pixel / thread) + a 6-pixel halo (window 3 + patch 3).
#include "nlm_direct.cuh"

extern "C" __global__ void __launch_bounds__(128) orion_nlm_direct_f4_128(orion_kargs a)
{
    ORION_PROBE(a);
    nlm_direct_body<32, 4, false>(a);
}
