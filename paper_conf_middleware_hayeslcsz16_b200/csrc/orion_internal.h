// orion_internal.h -- liborion internals shared by its translation units.
#pragma once
#include <atomic>
#include <memory>
#include <string>
#include <vector>

#include "../../include/orion.h"
#include "cuda_drv.h"
#include "orion_kargs.h"

namespace orion {

// ---- errors -------------------------------------------------------------------------------
orion_status fail(orion_status s, const std::string &msg);   // sets the thread-local message
orion_status cu_fail(CUresult r, const char *what);          // maps a driver error
#define ORION_CU(call)                                                   \
    do {                                                                 \
        CUresult _r = (call);                                            \
        if (_r != CUDA_SUCCESS) return ::orion::cu_fail(_r, #call);      \
    } while (0)
#define ORION_TRY(expr)                                                  \
    do {                                                                 \
        orion_status _s = (expr);                                        \
        if (_s != ORION_OK) return _s;                                   \
    } while (0)

extern std::atomic<long long> g_launches;
// Set while orion_tuner_capture records a graph: launches inside it are plain (no PDL attribute).
extern thread_local bool t_capturing;
// ... and whether its launches keep programmatic dependent launch (every captured launch
// independent: ORION_ARGS_INDEPENDENT), so the graph gets programmatic edges.
extern thread_local bool t_capture_pdl;

// The last kernel liborion enqueued on a stream: its orion_chain (tag) or nullptr for any other
// kernel.  A chained launch skips the grid-wide wait only behind its own chain's previous launch.
void note_stream_launch(CUstream s, const void *tag);
const void *last_stream_tag(CUstream s);

// Makes the primary context of `device` current on the calling thread (retaining it).
orion_status ensure_context(int device);

// ---- occupancy arithmetic (levels.cpp) ----------------------------------------------------
int limit_regs(const orion_device_limits &d, int T, int regs);
int limit_warps(const orion_device_limits &d, int T);
// carveout_pct < 0: the driver default (the calculator treats it as the maximum).
int limit_smem(const orion_device_limits &d, int smem_static, int smem_dyn, int carveout_pct);
int ctas_per_sm(const orion_device_limits &d, int T, int regs, int smem_static, int smem_dyn, int carveout_pct,
                int *limiter);
// Smallest padding realising exactly k CTAs/SM at `regs` registers (0 if already k); -1 if impossible.
int pad_for_level(const orion_device_limits &d, int T, int regs, int smem_static, int smem_need, int k,
                  int carveout_pct);
int carveout_pct_for_kb(const orion_device_limits &d, int kb);
int level_carveout_pct(const orion_device_limits &d, const orion_level &L);
// Per-SM shared-memory budget a carveout preference requests (pct < 0: the maximum).
int carveout_pref_bytes(const orion_device_limits &d, int pct);
// The unified L1 / shared-memory configurations (KB), ascending.
const int *carveout_configs_kb(int *n);

// ---- kernel registry + code generation (registry.cpp) -------------------------------------
enum KernelKind { K_KNN = 0, K_NLM = 1, K_STENCIL = 2, K_SRAD = 3 };

struct KernelDef {
    const char *id;
    int threads;            // T
    const char *entry;      // PTX entry name
    const char *module;     // embedded PTX module name
    int bx, by;             // CTA shape
    int tile_w, tile_h;     // output pixels per CTA (grid = ceil(W/tile_w) x ceil(rows/tile_h))
    int halo;               // rows/cols of input halo the kernel reads (3 KNN, 6 NLM, 1 stencil)
    int kind;               // KernelKind
    int smem_tile;          // 1: stages a (tile + halo) float4 tile in dynamic smem; 0: none
    int smem_bytes;         // > 0: explicit dynamic shared-memory need (overrides smem_tile)
    int width_align;        // > 1: the image width must be a multiple of this
    int steps_per_launch;   // stencil steps one launch performs (0 / 1 = one)
    int fanout;             // 1: the kernel's epilogue honours orion_args.fanout (store_out)
    int srad_stats;         // 1: SRAD with the ROI statistics fused (slots behind src / dst grids)
    int chain;              // 1: honours orion_args.chain (tile-level waits between launches)
    int dyn_need() const
    {
        if (smem_bytes > 0) return smem_bytes;
        return smem_tile ? (tile_w + 2 * halo) * (tile_h + 2 * halo) * 16 : 0;
    }
};

// Find by id and threads (0 = the id's default entry).
const KernelDef *find_kernel(const char *id, int threads);

struct CompiledVariant {
    std::vector<char> cubin;
    int regs = 0, spill_store = 0, spill_load = 0, stack_bytes = 0, static_smem = 0;
    std::string log;
};

// ptxas (the embedded nvPTXCompiler) on `def`'s PTX at register cap `cap` (0 = uncapped);
// memoised per (entry, cap).  Host-only: needs no GPU.
orion_status compile_variant(const KernelDef &def, int cap, std::shared_ptr<const CompiledVariant> *out);
// Loads a standalone (uncapped) module by name, e.g. "gen", on the current context.
orion_status load_aux_module(int device, const char *module, CUmodule *out);

}  // namespace orion

// Opaque handles.
// A chain of launches of one kernel family over one whole grid on one stream (orion.h).
struct orion_chain {
    int device = 0;
    const orion::KernelDef *def = nullptr;
    int width = 0, height = 0, gx = 0, gy = 0;
    CUdeviceptr flags = 0;          // gy x gx epochs of the last completed launch per tile
    unsigned epoch = 0;             // launches enqueued so far
    CUstream stream = nullptr;
    bool stream_set = false;
};
struct orion_variants {
    int device = 0;
    const orion::KernelDef *def = nullptr;
    orion_device_limits dev{};
    orion_kernel_resources res{};
    struct Var {
        orion_level planned{};
        orion_level realised{};
        std::shared_ptr<const orion::CompiledVariant> cv;
        CUmodule mod = nullptr;
        CUfunction fn = nullptr;
        int regs = 0, local_bytes = 0, verified = 0, dyn_bytes = 0, carveout_pct = -1;
    };
    std::vector<Var> vars;
};

struct orion_tuner;
