"""O1 -- occupancy calculator and feasible-level set.  TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline leg may import
this module; the product (liborion's ``orion_levels``) is an independent C++
implementation that shares no code with it.

Definition followed (plain, exact integer arithmetic):

* PAPER.md §2 Eq. (1), P:L121-L127:
  ``Occupancy = Min(Nreg/Vreg, Nsmem/Vsmem)/Smax`` "... the number of active
  threads needs to be rounded up to a multiple of thread block size, and the
  register partition needs to be aligned according to register bank size
  constraints ... We use the formula in NVIDIA occupancy calculator [19]".
  The calculator's rules for compute capability 10.0 are SURVEY.md §8(c) O1
  (register allocation per warp in 256-register units, split over 4
  sub-partitions; warp-slot, CTA-slot and shared-memory limits with 1 KB
  reserved per CTA in 128-byte units) -- DESIGN.md reading R-A9.
* Feasible levels ("generate code at all occupancy levels";
  reading R-A10): every k = 1..k_max CTAs/SM.  k is realised by a register cap
  R_k (P:L215 realising occupancy by bounding registers) and, below the
  register-determined level, by padding dynamic shared memory ("tune
  occupancy down by dynamically increasing shared memory usage per thread").

Pins (tests/test_oracle_occupancy.py): SURVEY Appendix A hand-worked tables,
NVIDIA's header-only ``cudaOccMaxActiveBlocksPerMultiprocessor`` (compiled from
/usr/local/cuda/include/cuda_occupancy.h, an independent implementation) over a
grid of (T, regs, smem), and the Kepler GTX680 sanity case of Fig. 1 (P:L91,
P:L713).
"""
from __future__ import annotations

from dataclasses import dataclass, asdict

LIM_REGS, LIM_SMEM, LIM_WARPS, LIM_BLOCKS = 1, 2, 4, 8


@dataclass(frozen=True)
class Device:
    cc_major: int = 10
    cc_minor: int = 0
    sm_count: int = 148
    warp_size: int = 32
    regs_per_sm: int = 65536
    regs_per_block: int = 65536
    max_regs_per_thread: int = 255
    reg_alloc_unit: int = 256          # registers per warp, allocation granularity
    num_subpartitions: int = 4
    max_threads_per_sm: int = 2048
    max_threads_per_block: int = 1024
    max_blocks_per_sm: int = 32
    smem_per_sm: int = 233472          # 228 KB (carveout 100 %)
    smem_per_block_optin: int = 232448  # 227 KB
    smem_reserved_per_block: int = 1024
    smem_alloc_unit: int = 128

    def as_dict(self):
        return asdict(self)


B200 = Device()
# GTX680 (Kepler GK104): 65536 regs/SM, 64 warps/SM; cc 3.0 has
# 16 CTAs/SM, 63 regs/thread max, warp-granular 256-register allocation, 4 schedulers.
GTX680 = Device(cc_major=3, cc_minor=0, sm_count=8, regs_per_sm=65536, regs_per_block=65536,
                max_regs_per_thread=63, reg_alloc_unit=256, num_subpartitions=4,
                max_threads_per_sm=2048, max_threads_per_block=1024, max_blocks_per_sm=16,
                smem_per_sm=49152, smem_per_block_optin=49152, smem_reserved_per_block=0,
                smem_alloc_unit=256)


def _ceil_div(a: int, b: int) -> int:
    return -(-a // b)


def _round_up(a: int, b: int) -> int:
    return _ceil_div(a, b) * b


def warps_per_cta(dev: Device, T: int) -> int:
    return _ceil_div(T, dev.warp_size)


def limit_warps(dev: Device, T: int) -> int:
    if T > dev.max_threads_per_block:
        return 0
    return (dev.max_threads_per_sm // dev.warp_size) // warps_per_cta(dev, T)


def limit_blocks(dev: Device) -> int:
    return dev.max_blocks_per_sm


def limit_regs(dev: Device, T: int, regs: int) -> int:
    """CTAs/SM allowed by the register file at `regs` registers/thread."""
    w = warps_per_cta(dev, T)
    if regs > dev.max_regs_per_thread:
        return 0
    if regs <= 0:
        return 1 << 30
    rpw = _round_up(regs * dev.warp_size, dev.reg_alloc_unit)
    if rpw * _round_up(w, dev.num_subpartitions) > dev.regs_per_block or rpw * w > dev.regs_per_block:
        return 0
    warps_per_sp = (dev.regs_per_sm // dev.num_subpartitions) // rpw
    return (warps_per_sp * dev.num_subpartitions) // w


def smem_alloc_per_cta(dev: Device, smem_static: int, smem_dyn: int) -> int:
    return _round_up(smem_static + dev.smem_reserved_per_block + smem_dyn, dev.smem_alloc_unit)


# Shared-memory / L1 carveout configurations of cc 10.0 in KB (the unified 256 KB array:
# what is not shared memory is L1).  The paper's small- vs large-cache configurations
# (P:L757-P:L761, Table 3) are two points of this axis on Fermi/Kepler.
CARVEOUT_KB = (0, 8, 16, 32, 64, 100, 132, 164, 196, 228)


def smem_config(dev: Device, nbytes: int) -> int | None:
    """Smallest carveout configuration (bytes) holding `nbytes`."""
    for kb in CARVEOUT_KB:
        c = min(kb * 1024, dev.smem_per_sm)
        if nbytes <= c:
            return c
    return None


def carveout_budget(dev: Device, carveout_pct: int | None) -> int:
    """Shared memory per SM a carveout preference asks for: pct of the maximum, rounded up
    to a configuration; None (the default) counts as the maximum."""
    if carveout_pct is None:
        return dev.smem_per_sm
    return smem_config(dev, carveout_pct * dev.smem_per_sm // 100)


def carveout_pct_for(dev: Device, kb: int) -> int:
    """Largest percentage that still rounds up to exactly `kb` KB."""
    return (kb * 1024 * 100) // dev.smem_per_sm


def limit_smem(dev: Device, smem_static: int, smem_dyn: int, carveout_pct: int | None = None) -> int:
    a = smem_alloc_per_cta(dev, smem_static, smem_dyn)
    if a > dev.smem_per_block_optin + dev.smem_reserved_per_block:
        return 0
    if a == 0:
        return 1 << 30
    budget = carveout_budget(dev, carveout_pct)
    if budget < a:                       # the driver raises the configuration to fit one CTA
        budget = smem_config(dev, a)
    return budget // a


def ctas_per_sm(dev: Device, T: int, regs: int, smem_static: int = 0, smem_dyn: int = 0,
                carveout_pct: int | None = None) -> int:
    """k = min(L_reg, L_warp, L_blk, L_smem) -- the calculator's answer."""
    return min(limit_regs(dev, T, regs), limit_warps(dev, T), limit_blocks(dev),
               limit_smem(dev, smem_static, smem_dyn, carveout_pct))


def limiter_mask(dev: Device, T: int, regs: int, smem_static: int, smem_dyn: int,
                 carveout_pct: int | None = None) -> int:
    k = ctas_per_sm(dev, T, regs, smem_static, smem_dyn, carveout_pct)
    m = 0
    if limit_regs(dev, T, regs) == k:
        m |= LIM_REGS
    if limit_smem(dev, smem_static, smem_dyn, carveout_pct) == k:
        m |= LIM_SMEM
    if limit_warps(dev, T) == k:
        m |= LIM_WARPS
    if limit_blocks(dev) == k:
        m |= LIM_BLOCKS
    return m


def occupancy(dev: Device, T: int, k: int) -> float:
    return k * warps_per_cta(dev, T) / (dev.max_threads_per_sm // dev.warp_size)


@dataclass(frozen=True)
class Level:
    ctas_per_sm: int
    warps_per_sm: int
    occupancy_permille: int
    reg_cap: int            # 0 = uncapped (the kernel's natural register count)
    smem_pad_bytes: int
    limiter: int
    carveout_kb: int = 0    # shared-memory configuration realising the level; 0 = driver's choice


REALISE_MAX_SMEM, REALISE_MIN_CARVEOUT = 0, 1


def reg_cap_for(dev: Device, T: int, natural: int, k: int, min_reg_cap: int = 16) -> int | None:
    """R_k: 0 (uncapped) if natural registers admit k CTAs, else the largest multiple
    of 8 below `natural` whose register limit admits k; None if none >= min_reg_cap."""
    if limit_regs(dev, T, natural) >= k:
        return 0
    r = ((natural - 1) // 8) * 8
    while r >= min_reg_cap:
        if limit_regs(dev, T, r) >= k:
            return r
        r -= 8
    return None


def pad_for(dev: Device, T: int, regs: int, smem_static: int, smem_need: int, k: int,
            carveout_pct: int | None = None) -> int | None:
    """Smallest extra dynamic shared memory making the CTA count exactly k (0 if already k)
    under the given carveout preference."""
    base = ctas_per_sm(dev, T, regs, smem_static, smem_need, carveout_pct)
    if base == k:
        return 0
    if base < k:
        return None
    budget = carveout_budget(dev, carveout_pct)
    a_k = _round_up(budget // (k + 1) + 1, dev.smem_alloc_unit)
    pad = a_k - dev.smem_reserved_per_block - smem_static - smem_need
    if pad < 0 or limit_smem(dev, smem_static, smem_need + pad, carveout_pct) != k:
        return None
    return pad


def realise(dev: Device, T: int, regs: int, smem_static: int, smem_need: int, k: int, mode: int):
    """(pad, carveout_kb) realising k CTAs/SM, or None.  MAX_SMEM: pad against the full
    228 KB (pinned only when a pad is needed).  MIN_CARVEOUT: the smallest configuration
    that still admits k CTAs, padded inside it -- the rest of the array stays L1."""
    if mode == REALISE_MAX_SMEM:
        pad = pad_for(dev, T, regs, smem_static, smem_need, k)
        if pad is None:
            return None
        return pad, (dev.smem_per_sm // 1024 if pad > 0 else 0)
    need_alloc = smem_alloc_per_cta(dev, smem_static, smem_need)
    for kb in CARVEOUT_KB:
        # a configuration smaller than one CTA would be raised by the driver: skip it so
        # carveout_kb names the configuration actually used
        if kb == 0 or kb * 1024 > dev.smem_per_sm or kb * 1024 < need_alloc:
            continue
        pct = carveout_pct_for(dev, kb)
        if carveout_budget(dev, pct) != kb * 1024:
            continue
        pad = pad_for(dev, T, regs, smem_static, smem_need, k, pct)
        if pad is not None:
            return pad, kb
    return None


def level_carveout_pct(dev: Device, lv: Level) -> int | None:
    return carveout_pct_for(dev, lv.carveout_kb) if lv.carveout_kb > 0 else None


def levels(dev: Device, T: int, natural_regs: int, smem_static: int = 0, smem_need: int = 0,
           min_reg_cap: int = 16, mode: int = REALISE_MAX_SMEM) -> list[Level]:
    """All feasible levels k = 1..k_max, ascending k."""
    out = []
    kmax_bound = min(limit_warps(dev, T), limit_blocks(dev), limit_smem(dev, smem_static, smem_need))
    for k in range(1, kmax_bound + 1):
        cap = reg_cap_for(dev, T, natural_regs, k, min_reg_cap)
        if cap is None:
            continue
        regs = natural_regs if cap == 0 else cap
        r = realise(dev, T, regs, smem_static, smem_need, k, mode)
        if r is None:
            continue
        pad, kb = r
        w = warps_per_cta(dev, T)
        maxw = dev.max_threads_per_sm // dev.warp_size
        pct = carveout_pct_for(dev, kb) if kb > 0 else None
        out.append(Level(ctas_per_sm=k, warps_per_sm=k * w,
                         occupancy_permille=(k * w * 1000) // maxw,
                         reg_cap=cap, smem_pad_bytes=pad,
                         limiter=limiter_mask(dev, T, regs, smem_static, smem_need + pad, pct),
                         carveout_kb=kb))
    return out


def original_level_index(lv: list[Level]) -> int:
    """The 'original' version: natural (uncapped) registers at the most CTAs
    they admit -- the unpadded level when padding is the only other limiter."""
    cands = [i for i, l in enumerate(lv) if l.reg_cap == 0]
    if not cands:
        raise ValueError("no uncapped level")
    return max(cands, key=lambda i: lv[i].ctas_per_sm)
