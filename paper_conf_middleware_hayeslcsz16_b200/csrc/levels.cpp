// levels.cpp -- occupancy arithmetic and the feasible-level set (orion_levels).
//
// PAPER.md §2 Eq. (1) (P:L121-P:L127): Occupancy = Min(Nreg/Vreg, Nsmem/Vsmem)/Smax,
// refined with the NVIDIA occupancy calculator's rounding rules ("the number of active
// threads needs to be rounded up to a multiple of thread block size, and the register
// partition needs to be aligned according to register bank size constraints").  For
// cc 10.0 those rules are: registers are granted per warp in `reg_alloc_unit` units and
// split evenly over the 4 SM sub-partitions; warps, CTA slots and shared memory (1 KB
// reserved per CTA, 128-byte units) each bound the CTA count.  The shared-memory budget
// per SM is the unified L1/shared carveout configuration: one of {0, 8, 16, 32, 64, 100,
// 132, 164, 196, 228} KB, chosen from the function's carveout preference (percent of the
// maximum, rounded UP to a configuration) and raised to fit one CTA when it is smaller.
// "Small cache vs large cache" (P:L757-P:L761, Table 3) is this axis on B200.
#include <algorithm>
#include <climits>

#include "orion_internal.h"

namespace orion {

static inline int ceil_div(int a, int b) { return (a + b - 1) / b; }
static inline int round_up(int a, int b) { return ceil_div(a, b) * b; }

static inline int warps_of(const orion_device_limits &d, int T) { return ceil_div(T, d.warp_size); }

static const int kCarveoutKB[] = {0, 8, 16, 32, 64, 100, 132, 164, 196, 228};

// Smallest carveout configuration (bytes) holding `bytes`; -1 above the maximum.
int smem_config_bytes(const orion_device_limits &d, long long bytes)
{
    for (int kb : kCarveoutKB) {
        const long long c = std::min<long long>((long long)kb * 1024, d.smem_per_sm);
        if (bytes <= c) return (int)c;
    }
    return -1;
}

// Per-SM shared-memory budget requested by a carveout preference (pct < 0: the default,
// which the calculator treats as the maximum).
int carveout_pref_bytes(const orion_device_limits &d, int pct)
{
    if (pct < 0) return d.smem_per_sm;
    return smem_config_bytes(d, (long long)pct * d.smem_per_sm / 100);
}

// The percentage whose rounded-up configuration is exactly `kb` KB.
int carveout_pct_for_kb(const orion_device_limits &d, int kb)
{
    if (kb <= 0) return 0;
    return (int)((long long)kb * 1024 * 100 / d.smem_per_sm);
}

int limit_warps(const orion_device_limits &d, int T)
{
    if (T <= 0 || T > d.max_threads_per_block) return 0;
    return (d.max_threads_per_sm / d.warp_size) / warps_of(d, T);
}

int limit_regs(const orion_device_limits &d, int T, int regs)
{
    if (regs > d.max_regs_per_thread) return 0;
    if (regs <= 0) return INT_MAX;
    const int w = warps_of(d, T);
    const int per_warp = round_up(regs * d.warp_size, d.reg_alloc_unit);
    // hardware check: allocation assumed on all sub-partitions at once; software check: plain sum
    if ((long long)per_warp * round_up(w, d.num_subpartitions) > d.regs_per_block) return 0;
    if ((long long)per_warp * w > d.regs_per_block) return 0;
    const int warps_per_subpartition = (d.regs_per_sm / d.num_subpartitions) / per_warp;
    return warps_per_subpartition * d.num_subpartitions / w;
}

int limit_smem(const orion_device_limits &d, int smem_static, int smem_dyn, int carveout_pct)
{
    const int alloc = round_up(smem_static + d.smem_reserved_per_block + smem_dyn, d.smem_alloc_unit);
    if (alloc > d.smem_per_block_optin + d.smem_reserved_per_block) return 0;
    if (alloc == 0) return INT_MAX;
    int budget = carveout_pref_bytes(d, carveout_pct);
    if (budget < alloc) budget = smem_config_bytes(d, alloc);   // raised to fit one CTA
    return budget / alloc;
}

int ctas_per_sm(const orion_device_limits &d, int T, int regs, int smem_static, int smem_dyn, int carveout_pct,
                int *limiter)
{
    const int lr = limit_regs(d, T, regs), lw = limit_warps(d, T), lb = d.max_blocks_per_sm,
              ls = limit_smem(d, smem_static, smem_dyn, carveout_pct);
    const int k = std::min(std::min(lr, lw), std::min(lb, ls));
    if (limiter) {
        *limiter = (lr == k ? ORION_LIM_REGS : 0) | (ls == k ? ORION_LIM_SMEM : 0) |
                   (lw == k ? ORION_LIM_WARPS : 0) | (lb == k ? ORION_LIM_BLOCKS : 0);
    }
    return k;
}

int pad_for_level(const orion_device_limits &d, int T, int regs, int smem_static, int smem_need, int k,
                  int carveout_pct)
{
    const int unpadded = ctas_per_sm(d, T, regs, smem_static, smem_need, carveout_pct, nullptr);
    if (unpadded == k) return 0;
    if (unpadded < k || k < 1) return -1;
    // smallest 128-byte-granular CTA allocation a with floor(budget / a) == k
    const int budget = carveout_pref_bytes(d, carveout_pct);
    const int alloc = round_up(budget / (k + 1) + 1, d.smem_alloc_unit);
    const int pad = alloc - d.smem_reserved_per_block - smem_static - smem_need;
    if (pad < 0) return -1;
    if (limit_smem(d, smem_static, smem_need + pad, carveout_pct) != k) return -1;
    return pad;
}

// R_k: 0 when the natural count admits k CTAs, else the largest multiple of 8 (one
// 256-register warp allocation unit) below natural that does; -1 if none >= min_cap.
static int reg_cap_for(const orion_device_limits &d, int T, int natural, int k, int min_cap)
{
    if (limit_regs(d, T, natural) >= k) return 0;
    for (int r = ((natural - 1) / 8) * 8; r >= min_cap; r -= 8)
        if (limit_regs(d, T, r) >= k) return r;
    return -1;
}

// Realise level k at `regs` registers: carveout configuration + padding.  Returns false if
// impossible.  MAX_SMEM: carveout pinned at the maximum when padding is needed, left to the
// driver otherwise.  MIN_CARVEOUT: the smallest configuration that can hold k CTAs, so the
// rest of the 256 KB unified array stays L1 cache.
bool realise(const orion_device_limits &d, int T, int regs, int smem_static, int smem_need, int k, int mode,
             int *pad, int *carveout_kb)
{
    if (mode == ORION_REALISE_MAX_SMEM) {
        const int p = pad_for_level(d, T, regs, smem_static, smem_need, k, -1);
        if (p < 0) return false;
        *pad = p;
        *carveout_kb = p > 0 ? d.smem_per_sm / 1024 : 0;
        return true;
    }
    const int need_alloc = round_up(smem_static + d.smem_reserved_per_block + smem_need, d.smem_alloc_unit);
    for (int kb : kCarveoutKB) {
        // configurations too small for one CTA would be raised by the driver: skip them so
        // carveout_kb names the configuration actually used
        if (kb == 0 || (long long)kb * 1024 > d.smem_per_sm || kb * 1024 < need_alloc) continue;
        const int pct = carveout_pct_for_kb(d, kb);
        if (carveout_pref_bytes(d, pct) != kb * 1024) continue;
        const int p = pad_for_level(d, T, regs, smem_static, smem_need, k, pct);
        if (p < 0) continue;
        *pad = p;
        *carveout_kb = kb;
        return true;
    }
    return false;
}

const int *carveout_configs_kb(int *n)
{
    *n = (int)(sizeof kCarveoutKB / sizeof kCarveoutKB[0]);
    return kCarveoutKB;
}

int level_carveout_pct(const orion_device_limits &d, const orion_level &L)
{
    return L.carveout_kb > 0 ? carveout_pct_for_kb(d, L.carveout_kb) : -1;
}

}  // namespace orion

using namespace orion;

extern "C" {

orion_status orion_b200_limits(orion_device_limits *o)
{
    if (!o) return fail(ORION_E_INVALID, "orion_b200_limits: NULL");
    *o = orion_device_limits{10, 0, 148, 32, 65536, 65536, 255, 256, 4, 2048, 1024, 32, 233472, 232448, 1024, 128};
    return ORION_OK;
}

orion_status orion_query_limits(int device, orion_device_limits *o)
{
    if (!o) return fail(ORION_E_INVALID, "orion_query_limits: NULL");
    ORION_TRY(ensure_context(device));
    const Driver &D = drv();
    CUdevice dev;
    ORION_CU(D.cuDeviceGet(&dev, device));
    auto attr = [&](CUdevice_attribute a, int *v) { return D.cuDeviceGetAttribute(v, a, dev); };
    ORION_CU(attr(CU_DEVICE_ATTRIBUTE_COMPUTE_CAPABILITY_MAJOR, &o->cc_major));
    ORION_CU(attr(CU_DEVICE_ATTRIBUTE_COMPUTE_CAPABILITY_MINOR, &o->cc_minor));
    ORION_CU(attr(CU_DEVICE_ATTRIBUTE_MULTIPROCESSOR_COUNT, &o->sm_count));
    ORION_CU(attr(CU_DEVICE_ATTRIBUTE_WARP_SIZE, &o->warp_size));
    ORION_CU(attr(CU_DEVICE_ATTRIBUTE_MAX_REGISTERS_PER_MULTIPROCESSOR, &o->regs_per_sm));
    ORION_CU(attr(CU_DEVICE_ATTRIBUTE_MAX_REGISTERS_PER_BLOCK, &o->regs_per_block));
    ORION_CU(attr(CU_DEVICE_ATTRIBUTE_MAX_THREADS_PER_MULTIPROCESSOR, &o->max_threads_per_sm));
    ORION_CU(attr(CU_DEVICE_ATTRIBUTE_MAX_THREADS_PER_BLOCK, &o->max_threads_per_block));
    ORION_CU(attr(CU_DEVICE_ATTRIBUTE_MAX_BLOCKS_PER_MULTIPROCESSOR, &o->max_blocks_per_sm));
    ORION_CU(attr(CU_DEVICE_ATTRIBUTE_MAX_SHARED_MEMORY_PER_MULTIPROCESSOR, &o->smem_per_sm));
    ORION_CU(attr(CU_DEVICE_ATTRIBUTE_MAX_SHARED_MEMORY_PER_BLOCK_OPTIN, &o->smem_per_block_optin));
    ORION_CU(attr(CU_DEVICE_ATTRIBUTE_RESERVED_SHARED_MEMORY_PER_BLOCK, &o->smem_reserved_per_block));
    // Not exposed as attributes: the cc >= 7 calculator constants (cuda_occupancy.h).
    o->max_regs_per_thread = 255;
    o->reg_alloc_unit = 256;
    o->num_subpartitions = 4;
    o->smem_alloc_unit = 128;
    return ORION_OK;
}

orion_status orion_ctas_per_sm(const orion_device_limits *dev, int T, int regs, int smem_static, int smem_dyn,
                               int *ctas, int *limiter)
{
    return orion_ctas_per_sm_carveout(dev, T, regs, smem_static, smem_dyn, -1, ctas, limiter);
}

orion_status orion_ctas_per_sm_carveout(const orion_device_limits *dev, int T, int regs, int smem_static,
                                        int smem_dyn, int carveout_pct, int *ctas, int *limiter)
{
    if (!dev || !ctas || T <= 0 || regs < 0 || smem_static < 0 || smem_dyn < 0 || carveout_pct > 100)
        return fail(ORION_E_INVALID, "orion_ctas_per_sm: bad argument");
    *ctas = ctas_per_sm(*dev, T, regs, smem_static, smem_dyn, carveout_pct < 0 ? -1 : carveout_pct, limiter);
    return ORION_OK;
}

orion_status orion_levels(const orion_device_limits *dev, const orion_kernel_resources *res, orion_level *out,
                          int capacity, int *n_out)
{
    return orion_levels_ex(dev, res, ORION_REALISE_MAX_SMEM, out, capacity, n_out);
}

orion_status orion_levels_ex(const orion_device_limits *dev, const orion_kernel_resources *res, int mode,
                             orion_level *out, int capacity, int *n_out)
{
    if (!dev || !res || !n_out || capacity < 0 || (capacity > 0 && !out) ||
        (mode != ORION_REALISE_MAX_SMEM && mode != ORION_REALISE_MIN_CARVEOUT))
        return fail(ORION_E_INVALID, "orion_levels: bad argument");
    const orion_device_limits &d = *dev;
    const int T = res->block_threads;
    if (T <= 0 || T > d.max_threads_per_block || res->regs_per_thread <= 0 ||
        res->regs_per_thread > d.max_regs_per_thread || res->static_smem_bytes < 0 || res->dyn_smem_bytes < 0)
        return fail(ORION_E_INVALID, "orion_levels: bad kernel resources");
    const int min_cap = res->min_reg_cap > 0 ? res->min_reg_cap : 16;
    const int w = (T + d.warp_size - 1) / d.warp_size;
    const int max_warps = d.max_threads_per_sm / d.warp_size;
    const int bound = std::min(std::min(limit_warps(d, T), d.max_blocks_per_sm),
                               limit_smem(d, res->static_smem_bytes, res->dyn_smem_bytes, -1));
    std::vector<orion_level> lv;
    for (int k = 1; k <= bound; ++k) {
        const int cap = reg_cap_for(d, T, res->regs_per_thread, k, min_cap);
        if (cap < 0) continue;
        const int regs = cap == 0 ? res->regs_per_thread : cap;
        int pad = 0, kb = 0;
        if (!realise(d, T, regs, res->static_smem_bytes, res->dyn_smem_bytes, k, mode, &pad, &kb)) continue;
        orion_level L;
        L.ctas_per_sm = k;
        L.warps_per_sm = k * w;
        L.occupancy_permille = (k * w * 1000) / max_warps;
        L.reg_cap = cap;
        L.smem_pad_bytes = pad;
        L.carveout_kb = kb;
        ctas_per_sm(d, T, regs, res->static_smem_bytes, res->dyn_smem_bytes + pad, level_carveout_pct(d, L),
                    &L.limiter);
        lv.push_back(L);
    }
    *n_out = (int)lv.size();
    if ((int)lv.size() > capacity) return fail(ORION_E_CAPACITY, "orion_levels: capacity too small");
    std::copy(lv.begin(), lv.end(), out);
    return ORION_OK;
}

}  // extern "C"
