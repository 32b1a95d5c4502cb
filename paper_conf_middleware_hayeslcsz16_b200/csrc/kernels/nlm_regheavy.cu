// nlm_regheavy.cu -- the register-heavy NLM variant of config C4 (see nlm_direct.cu):
// the centre patch lives in registers across all 49 window offsets, so the natural
// register demand is far above 32 and register caps trade spills for occupancy
// (Table 2 "Reg" column P:L725).
#include "nlm_direct.cuh"

extern "C" __global__ void __launch_bounds__(128) orion_nlm_regheavy_f4_128(orion_kargs a)
{
    ORION_PROBE(a);
    nlm_direct_body<32, 4, true>(a);
}
extern "C" __global__ void __launch_bounds__(64) orion_nlm_regheavy_f4_64(orion_kargs a)
{
    ORION_PROBE(a);
    nlm_direct_body<8, 8, true>(a);
}
