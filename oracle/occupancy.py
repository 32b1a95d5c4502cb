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


def limit_smem(dev: Device, smem_static: int, smem_dyn: int) -> int:
    a = smem_alloc_per_cta(dev, smem_static, smem_dyn)
    if a > dev.smem_per_block_optin + dev.smem_reserved_per_block:
        return 0
    if a == 0:
        return 1 << 30
    return dev.smem_per_sm // a


def ctas_per_sm(dev: Device, T: int, regs: int, smem_static: int = 0, smem_dyn: int = 0) -> int:
    """k = min(L_reg, L_warp, L_blk, L_smem) -- the calculator's answer."""
    return min(limit_regs(dev, T, regs), limit_warps(dev, T), limit_blocks(dev),
               limit_smem(dev, smem_static, smem_dyn))


def limiter_mask(dev: Device, T: int, regs: int, smem_static: int, smem_dyn: int) -> int:
    k = ctas_per_sm(dev, T, regs, smem_static, smem_dyn)
    m = 0
    if limit_regs(dev, T, regs) == k:
        m |= LIM_REGS
    if limit_smem(dev, smem_static, smem_dyn) == k:
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


def pad_for(dev: Device, T: int, regs: int, smem_static: int, smem_need: int, k: int) -> int | None:
    """Smallest extra dynamic shared memory making the CTA count exactly k (0 if already k)."""
    base = min(limit_regs(dev, T, regs), limit_warps(dev, T), limit_blocks(dev),
               limit_smem(dev, smem_static, smem_need))
    if base == k:
        return 0
    if base < k:
        return None
    a_k = _round_up(dev.smem_per_sm // (k + 1) + 1, dev.smem_alloc_unit)
    pad = a_k - dev.smem_reserved_per_block - smem_static - smem_need
    if pad < 0 or limit_smem(dev, smem_static, smem_need + pad) != k:
        return None
    return pad


def levels(dev: Device, T: int, natural_regs: int, smem_static: int = 0, smem_need: int = 0,
           min_reg_cap: int = 16) -> list[Level]:
    """All feasible levels k = 1..k_max, ascending k."""
    out = []
    kmax_bound = min(limit_warps(dev, T), limit_blocks(dev), limit_smem(dev, smem_static, smem_need))
    for k in range(1, kmax_bound + 1):
        cap = reg_cap_for(dev, T, natural_regs, k, min_reg_cap)
        if cap is None:
            continue
        regs = natural_regs if cap == 0 else cap
        pad = pad_for(dev, T, regs, smem_static, smem_need, k)
        if pad is None:
            continue
        w = warps_per_cta(dev, T)
        maxw = dev.max_threads_per_sm // dev.warp_size
        out.append(Level(ctas_per_sm=k, warps_per_sm=k * w,
                         occupancy_permille=(k * w * 1000) // maxw,
                         reg_cap=cap, smem_pad_bytes=pad,
                         limiter=limiter_mask(dev, T, regs, smem_static, smem_need + pad)))
    return out


def original_level_index(lv: list[Level]) -> int:
    """The 'original' version: uncapped registers, no padding."""
    for i, l in enumerate(lv):
        if l.reg_cap == 0 and l.smem_pad_bytes == 0:
            return i
    raise ValueError("no uncapped, unpadded level")
