// drv.cpp -- run-time binding of the CUDA driver, error plumbing, context handling.
#include <dlfcn.h>

#include <cstdio>
#include <map>
#include <mutex>

#include "orion_internal.h"

namespace orion {

#define ORION_STR2(x) #x
#define ORION_STR(x) ORION_STR2(x)

const Driver &drv()
{
    static Driver d;
    static std::once_flag once;
    std::call_once(once, [] {
        void *h = dlopen("libcuda.so.1", RTLD_NOW | RTLD_LOCAL);
        if (!h) {
            d.why = std::string("CUDA driver not available: ") + dlerror();
            return;
        }
#define ORION_LOAD(f)                                                        \
    d.f = reinterpret_cast<decltype(&::f)>(dlsym(h, ORION_STR(f)));          \
    if (!d.f) {                                                              \
        d.why = "libcuda.so.1 lacks " ORION_STR(f);                          \
        return;                                                              \
    }
        ORION_CU_FUNCS(ORION_LOAD)
#undef ORION_LOAD
        CUresult r = d.cuInit(0);
        if (r != CUDA_SUCCESS) {
            char buf[64];
            std::snprintf(buf, sizeof buf, "cuInit failed (%d)", (int)r);
            d.why = buf;
            return;
        }
        d.ok = true;
    });
    return d;
}

static thread_local std::string t_last_error;
std::atomic<long long> g_launches{0};
thread_local bool t_capturing = false;
thread_local bool t_capture_pdl = false;

orion_status fail(orion_status s, const std::string &msg)
{
    t_last_error = msg;
    return s;
}

orion_status cu_fail(CUresult r, const char *what)
{
    const char *name = nullptr, *str = nullptr;
    if (drv().ok) {
        drv().cuGetErrorName(r, &name);
        drv().cuGetErrorString(r, &str);
    }
    return fail(ORION_E_CUDA, std::string(what) + ": " + (name ? name : "?") + " (" + (str ? str : "") + ")");
}

orion_status ensure_context(int device)
{
    const Driver &d = drv();
    if (!d.ok) return fail(ORION_E_CUDA, d.why);
    CUcontext cur = nullptr;
    ORION_CU(d.cuCtxGetCurrent(&cur));
    if (cur) {
        CUdevice cd;
        ORION_CU(d.cuCtxGetDevice(&cd));
        CUdevice want;
        ORION_CU(d.cuDeviceGet(&want, device));
        if (cd == want) return ORION_OK;
    }
    // each device's primary context is retained ONCE per process (the reference is held for
    // the library's lifetime and released at unload); later switches reuse the cached handle
    static std::mutex mu;
    static std::map<int, CUcontext> retained;
    CUcontext ctx = nullptr;
    {
        std::lock_guard<std::mutex> lk(mu);
        auto it = retained.find(device);
        if (it != retained.end()) {
            ctx = it->second;
        } else {
            CUdevice dev;
            ORION_CU(d.cuDeviceGet(&dev, device));
            ORION_CU(d.cuDevicePrimaryCtxRetain(&ctx, dev));
            retained[device] = ctx;
        }
    }
    ORION_CU(d.cuCtxSetCurrent(ctx));
    return ORION_OK;
}

}  // namespace orion

extern "C" {

const char *orion_last_error(void) { return orion::t_last_error.c_str(); }

const char *orion_status_str(orion_status s)
{
    switch (s) {
    case ORION_OK: return "ORION_OK";
    case ORION_E_INVALID: return "ORION_E_INVALID";
    case ORION_E_CAPACITY: return "ORION_E_CAPACITY";
    case ORION_E_INFEASIBLE: return "ORION_E_INFEASIBLE";
    case ORION_E_COMPILE: return "ORION_E_COMPILE";
    case ORION_E_CUDA: return "ORION_E_CUDA";
    case ORION_E_OCCUPANCY_MISMATCH: return "ORION_E_OCCUPANCY_MISMATCH";
    case ORION_E_STATE: return "ORION_E_STATE";
    default: return "ORION_E_UNKNOWN";
    }
}

long long orion_launch_count(void) { return orion::g_launches.load(); }

const char *orion_version(void) { return "liborion 0.1 (sm_100a)"; }

}  // extern "C"
