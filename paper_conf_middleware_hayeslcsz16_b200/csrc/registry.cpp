// registry.cpp -- the kernel families liborion knows, and their code generation.
//
// The paper's compiler realises an occupancy level by re-allocating registers in SASS
// (P:L213-P:L229, P:L697-P:L707).  On sm_100a ptxas owns register allocation, so a
// level's register budget is realised the way NVIDIA's toolchain exposes it: each
// kernel is compiled ONCE to PTX when the library is built (nvcc -arch=compute_100a
// -fmad=false; the PTX is embedded in liborion.so), and `orion_build_variants`
// assembles that PTX to an sm_100a cubin once per distinct register cap with the
// embedded ptxas (nvPTXCompiler, --maxrregcount=R).  One PTX + explicit .rn arithmetic
// => every variant computes bit-identical results; only resources differ.
#include <nvPTXCompiler.h>

#include <cstdio>
#include <cstring>
#include <map>
#include <mutex>
#include <sstream>

#include "orion_internal.h"

// Generated at build time (build.py): the PTX of every kernel family, NUL-terminated.
extern "C" const char liborion_ptx_knn[];
extern "C" const char liborion_ptx_nlm_box[];
extern "C" const char liborion_ptx_nlm_direct[];
extern "C" const char liborion_ptx_nlm_regheavy[];
extern "C" const char liborion_ptx_hotspot[];
extern "C" const char liborion_ptx_gen[];
extern "C" const char liborion_ptx_srad[];
extern "C" const char liborion_ptx_nlm_boxw[];

namespace orion {

static const char *module_ptx(const char *module)
{
    if (!std::strcmp(module, "knn")) return liborion_ptx_knn;
    if (!std::strcmp(module, "nlm_box")) return liborion_ptx_nlm_box;
    if (!std::strcmp(module, "nlm_direct")) return liborion_ptx_nlm_direct;
    if (!std::strcmp(module, "nlm_regheavy")) return liborion_ptx_nlm_regheavy;
    if (!std::strcmp(module, "hotspot")) return liborion_ptx_hotspot;
    if (!std::strcmp(module, "gen")) return liborion_ptx_gen;
    if (!std::strcmp(module, "srad")) return liborion_ptx_srad;
    if (!std::strcmp(module, "nlm_boxw")) return liborion_ptx_nlm_boxw;
    return nullptr;
}

// id, T, entry, module, bx, by, tile_w, tile_h, halo, kind, smem_tile, smem_bytes.  The first row of
// each id is its default CTA size.
static const KernelDef kKernels[] = {
    {"knn_f4", 128, "orion_knn_f4_128", "knn", 32, 4, 32, 16, 3, K_KNN, 1, 0, 1, 1, 1},
    {"knn_f4", 256, "orion_knn_f4_256", "knn", 32, 8, 32, 32, 3, K_KNN, 1, 0, 1, 1, 1},
    {"knn_f4", 64, "orion_knn_f4_64", "knn", 8, 8, 8, 32, 3, K_KNN, 1, 0, 1, 1, 1},
    // one pixel per thread: small (launch-bound) frames
    {"knn_f4_p1", 128, "orion_knn1_f4_128", "knn", 32, 4, 32, 4, 3, K_KNN, 1, 0, 1, 1, 1},
    {"knn_f4_p1", 64, "orion_knn1_f4_64", "knn", 8, 8, 8, 8, 3, K_KNN, 1, 0, 1, 1, 1},
    // 16 threads per pixel, 8 pixels of one row per CTA
    {"knn_f4_t16", 128, "orion_knn16_f4_128", "knn", 128, 1, 8, 1, 3, K_KNN, 0, 0, 1, 1, 1},
    // nlm_box: 3 planar (122+18) x (23+12) fp32 planes (pitch 141) + 3 H_o buffers of 32 x 129
    // floats, 3 offset pairs per pass (2 CTAs/SM)
    {"nlm_f4", 128, "orion_nlm_box3_f4_128", "nlm_box", 128, 1, 122, 23, 6, K_NLM, 0,
     3 * 35 * 141 * 4 + 3 * 32 * 129 * 4, 1, 1, 1},
    // 128-column tiles: planes (128+20) x 35 (pitch 149) + 3 H buffers of 32 x 137 floats -- the
    // C2 / C5 default
    {"nlm_f4_w", 128, "orion_nlm_boxw3_f4_128", "nlm_boxw", 128, 1, 128, 23, 6, K_NLM, 0,
     3 * 35 * 149 * 4 + 3 * 32 * 137 * 4, 1, 1, 1},
    // the direct 2401-term definition (cross-check form), and the register-heavy C4 kernel
    {"nlm_f4_direct", 128, "orion_nlm_direct_f4_128", "nlm_direct", 32, 4, 32, 4, 6, K_NLM, 1, 0},
    {"nlm_f4_regheavy", 128, "orion_nlm_regheavy_f4_128", "nlm_regheavy", 32, 4, 32, 4, 6, K_NLM, 1, 0},
    {"nlm_f4_regheavy", 64, "orion_nlm_regheavy_f4_64", "nlm_regheavy", 8, 8, 8, 8, 6, K_NLM, 1, 0},
    {"hotspot_f32", 256, "orion_hotspot_f32_256", "hotspot", 32, 8, 128, 128, 1, K_STENCIL, 0, 0},
    {"hotspot_f32", 128, "orion_hotspot_f32_128", "hotspot", 32, 4, 128, 64, 1, K_STENCIL, 0, 0},
    // two steps per launch (temporal blocking) with whole halo lanes: 120 output columns per warp, 6-slot ring of
    // 8 warps x 6 x 256 floats
    {"hotspot2h_f32", 256, "orion_hotspot2h_f32_256", "hotspot", 32, 8, 120, 256, 2, K_STENCIL, 0, 8 * 6 * 256 * 4, 4, 2},
    // four steps per launch, whole halo lanes: the same 120-column warps walking 128-row strips as
    // a 4-stage register pipeline; 9-slot ring of 8 warps x 9 x 256 floats; reads 4 rows beyond;
    // fan-out = the halo exchange of a row-sharded grid (first / last 4 rows to the neighbours);
    // chainable (orion_chain: tile-level waits between consecutive launches)
    {"hotspot4h_f32", 256, "orion_hotspot4h_f32_256", "hotspot", 32, 8, 120, 1024, 4, K_STENCIL, 0, 8 * 9 * 256 * 4, 4, 4,
     1, 0, 1},
    // srad: J tile (32+3)^2 + coefficient tile (32+1)^2 floats; reads 2 rows below the tile
    {"srad_f32_tile", 256, "orion_srad_f32_256", "srad", 32, 8, 32, 32, 2, K_SRAD, 0, (35 * 35 + 33 * 33) * 4},
    // srad, register-sliding: 124 x 128 tile; float4 lanes (width % 4 == 0) or scalar lanes;
    // rows stream through a 4-slot cp.async ring per warp (8 x 4 x 132 floats)
    {"srad_f32", 256, "orion_srad4_f32_256", "srad", 32, 8, 124, 256, 2, K_SRAD, 0, 8 * 6 * 132 * 4},
    // srad, halo lanes: 120 x 336 tile, width % 4 == 0; 6-slot ring of 8 warps x 6 x 128 floats
    {"srad_f32h", 256, "orion_srad4h_f32_256", "srad", 32, 8, 120, 8 * 42, 2, K_SRAD, 0, 8 * 6 * 128 * 4, 4},
    // the same with the ROI statistics fused: q0sqr from the slots behind src, the output ROI's
    // slots written behind dst (no statistics kernel per iteration; whole grids); chainable
    {"srad_f32hs", 256, "orion_srad4hs_f32_256", "srad", 32, 8, 120, 8 * 42, 2, K_SRAD, 0, 8 * 6 * 128 * 4, 4, 0, 0, 1,
     1},
};

const KernelDef *find_kernel(const char *id, int threads)
{
    if (!id) return nullptr;
    for (const KernelDef &k : kKernels)
        if (!std::strcmp(k.id, id) && (threads == 0 || threads == k.threads)) return &k;
    return nullptr;
}

static void parse_ptxas_log(const std::string &log, CompiledVariant &cv)
{
    std::istringstream in(log);
    std::string line;
    while (std::getline(in, line)) {
        int a, b, c;
        const char *p;
        if ((p = std::strstr(line.c_str(), "bytes stack frame")) != nullptr) {
            if (std::sscanf(line.c_str() + line.find_first_of("0123456789"),
                            "%d bytes stack frame, %d bytes spill stores, %d bytes spill loads", &a, &b, &c) == 3) {
                cv.stack_bytes = a;
                cv.spill_store = b;
                cv.spill_load = c;
            }
        }
        if ((p = std::strstr(line.c_str(), "Used ")) != nullptr) {
            if (std::sscanf(p, "Used %d registers", &a) == 1) cv.regs = a;
            const char *s = std::strstr(p, "bytes smem");
            if (s) {
                const char *q = s;
                while (q > p && q[-1] == ' ') --q;
                while (q > p && q[-1] >= '0' && q[-1] <= '9') --q;
                cv.static_smem = std::atoi(q);
            }
        }
    }
}

orion_status compile_variant(const KernelDef &def, int cap, std::shared_ptr<const CompiledVariant> *out)
{
    static std::mutex mu;
    static std::map<std::pair<std::string, int>, std::shared_ptr<const CompiledVariant>> cache;
    const auto key = std::make_pair(std::string(def.entry), cap);
    {
        std::lock_guard<std::mutex> g(mu);
        auto it = cache.find(key);
        if (it != cache.end()) {
            *out = it->second;
            return ORION_OK;
        }
    }
    const char *ptx0 = module_ptx(def.module);
    if (!ptx0) return fail(ORION_E_INVALID, std::string("no PTX module ") + def.module);
    // The register budget of a level is a per-entry PTX performance directive: `.maxnreg R`
    // is inserted after the entry's `.maxntid` (its __launch_bounds__, which would make
    // ptxas ignore a global --maxrregcount).  Everything else in the PTX is untouched.
    std::string ptx(ptx0);
    if (cap > 0) {
        const std::string ent = std::string(".entry ") + def.entry + "(";
        size_t at = ptx.find(ent);
        size_t mt = at == std::string::npos ? at : ptx.find(".maxntid", at);
        size_t body = at == std::string::npos ? at : ptx.find("\n{", at);
        if (mt == std::string::npos || body == std::string::npos || mt > body)
            return fail(ORION_E_COMPILE, std::string("no .maxntid directive for ") + def.entry);
        size_t eol = ptx.find('\n', mt);
        ptx.insert(eol + 1, ".maxnreg " + std::to_string(cap) + "\n");
    }
    nvPTXCompilerHandle h = nullptr;
    if (nvPTXCompilerCreate(&h, ptx.size(), ptx.c_str()) != NVPTXCOMPILE_SUCCESS)
        return fail(ORION_E_COMPILE, "nvPTXCompilerCreate failed");
    std::string entry = std::string("--entry=") + def.entry;
    std::vector<const char *> opts = {"--gpu-name=sm_100a", "--verbose", "-O3", "--generate-line-info",
                                      entry.c_str()};
    nvPTXCompileResult r = nvPTXCompilerCompile(h, (int)opts.size(), opts.data());
    auto cv = std::make_shared<CompiledVariant>();
    size_t n = 0;
    if (nvPTXCompilerGetInfoLogSize(h, &n) == NVPTXCOMPILE_SUCCESS && n) {
        cv->log.resize(n);
        nvPTXCompilerGetInfoLog(h, &cv->log[0]);
    }
    if (r != NVPTXCOMPILE_SUCCESS) {
        std::string err;
        if (nvPTXCompilerGetErrorLogSize(h, &n) == NVPTXCOMPILE_SUCCESS && n) {
            err.resize(n);
            nvPTXCompilerGetErrorLog(h, &err[0]);
        }
        nvPTXCompilerDestroy(&h);
        return fail(ORION_E_COMPILE, std::string("ptxas failed for ") + def.entry + " cap " + std::to_string(cap) +
                                         ": " + err);
    }
    if (nvPTXCompilerGetCompiledProgramSize(h, &n) != NVPTXCOMPILE_SUCCESS) {
        nvPTXCompilerDestroy(&h);
        return fail(ORION_E_COMPILE, "nvPTXCompilerGetCompiledProgramSize failed");
    }
    cv->cubin.resize(n);
    nvPTXCompilerGetCompiledProgram(h, cv->cubin.data());
    nvPTXCompilerDestroy(&h);
    parse_ptxas_log(cv->log, *cv);
    std::lock_guard<std::mutex> g(mu);
    auto &slot = cache[key];
    if (!slot) slot = cv;
    *out = slot;
    return ORION_OK;
}

orion_status load_aux_module(int device, const char *module, CUmodule *out)
{
    static std::mutex mu;
    static std::map<std::pair<int, std::string>, CUmodule> mods;
    ORION_TRY(ensure_context(device));
    std::lock_guard<std::mutex> g(mu);
    auto key = std::make_pair(device, std::string(module));
    auto it = mods.find(key);
    if (it != mods.end()) {
        *out = it->second;
        return ORION_OK;
    }
    const char *ptx = module_ptx(module);
    if (!ptx) return fail(ORION_E_INVALID, std::string("no PTX module ") + module);
    nvPTXCompilerHandle h = nullptr;
    if (nvPTXCompilerCreate(&h, std::strlen(ptx), ptx) != NVPTXCOMPILE_SUCCESS)
        return fail(ORION_E_COMPILE, "nvPTXCompilerCreate failed");
    const char *opts[] = {"--gpu-name=sm_100a", "-O3"};
    if (nvPTXCompilerCompile(h, 2, opts) != NVPTXCOMPILE_SUCCESS) {
        nvPTXCompilerDestroy(&h);
        return fail(ORION_E_COMPILE, std::string("ptxas failed for module ") + module);
    }
    size_t n = 0;
    nvPTXCompilerGetCompiledProgramSize(h, &n);
    std::vector<char> cubin(n);
    nvPTXCompilerGetCompiledProgram(h, cubin.data());
    nvPTXCompilerDestroy(&h);
    CUmodule m;
    ORION_CU(drv().cuModuleLoadData(&m, cubin.data()));
    mods[key] = m;
    *out = m;
    return ORION_OK;
}

}  // namespace orion

using namespace orion;

extern "C" {

orion_status orion_kernel_probe(const char *kernel_id, int block_threads, orion_kernel_resources *out)
{
    if (!out) return fail(ORION_E_INVALID, "orion_kernel_probe: NULL");
    const KernelDef *def = find_kernel(kernel_id, block_threads);
    if (!def) return fail(ORION_E_INVALID, std::string("unknown kernel ") + (kernel_id ? kernel_id : "(null)"));
    std::shared_ptr<const CompiledVariant> cv;
    ORION_TRY(compile_variant(*def, 0, &cv));
    out->block_threads = def->threads;
    out->regs_per_thread = cv->regs;
    out->static_smem_bytes = cv->static_smem;
    out->dyn_smem_bytes = def->dyn_need();
    out->min_reg_cap = 16;
    return ORION_OK;
}

orion_status orion_compile_info(const char *kernel_id, int block_threads, int reg_cap, int *regs, int *spill_st,
                                int *spill_ld, int *local_bytes)
{
    const KernelDef *def = find_kernel(kernel_id, block_threads);
    if (!def || reg_cap < 0 || reg_cap > 255) return fail(ORION_E_INVALID, "orion_compile_info: bad argument");
    std::shared_ptr<const CompiledVariant> cv;
    ORION_TRY(compile_variant(*def, reg_cap, &cv));
    if (regs) *regs = cv->regs;
    if (spill_st) *spill_st = cv->spill_store;
    if (spill_ld) *spill_ld = cv->spill_load;
    if (local_bytes) *local_bytes = cv->stack_bytes;
    return ORION_OK;
}

}  // extern "C"
