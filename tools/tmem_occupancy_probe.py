"""Does a kernel that allocates tensor memory (tcgen05.alloc) get more than one CTA per SM?
Compiles tools/tmem_occupancy_probe.cu for sm_100a and asks the driver's occupancy API for each
entry at T = 32 with no shared memory.  Measured on B200 (CUDA 12.9, driver 580): the plain
kernel 32 CTAs/SM, every tcgen05.alloc kernel 1 -- whatever the column count (32 / 128 / 512).
The residency probe of the NLM kernel with a 128-column allocation measured 1 as well (DESIGN.md
section 10).  Usage (on a GPU box): python tools/tmem_occupancy_probe.py"""
import os
import subprocess
import tempfile

from cuda.bindings import driver as cu

HERE = os.path.dirname(os.path.abspath(__file__))
with tempfile.TemporaryDirectory() as d:
    cubin = os.path.join(d, "probe.cubin")
    subprocess.check_call(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-cubin", "-o", cubin,
                           os.path.join(HERE, "tmem_occupancy_probe.cu")])
    cu.cuInit(0)
    _, dev = cu.cuDeviceGet(0)
    _, ctx = cu.cuDevicePrimaryCtxRetain(dev)
    cu.cuCtxSetCurrent(ctx)
    _, mod = cu.cuModuleLoadData(open(cubin, "rb").read())
    for e in (b"k_plain", b"k_tm32", b"k_tm128", b"k_tm512"):
        _, f = cu.cuModuleGetFunction(mod, e)
        _, n = cu.cuOccupancyMaxActiveBlocksPerMultiprocessor(f, 32, 0)
        print(e.decode(), "CTAs/SM at T = 32:", n, flush=True)
