// variants.cpp -- the multi-version binary (orion_build_variants), realising a level at
// launch (orion_launch), the exhaustive sweep, and the synthetic-input generators.
//
// Realising occupancy level k on sm_100a (§3.2 P:L213-P:L229 realises it by
// bounding registers and shared memory per thread; P:L649 lowers it "by dynamically
// increasing shared memory usage per thread"):
//   registers      -> the variant's cubin was assembled with --maxrregcount=R_k;
//   shared memory  -> the launch requests the kernel's own need + pad_k bytes of dynamic
//                     shared memory, pad_k recomputed from the ACTUAL register count, with
//                     the shared-memory carveout pinned at 100 % whenever pad_k > 0 so the
//                     per-SM budget the pad divides is the full 228 KB;
//   verification   -> cuOccupancyMaxActiveBlocksPerMultiprocessor must report exactly k.
#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <unordered_map>
#include <string>
#include <vector>

#include <atomic>

#include "orion_internal.h"

using namespace orion;

// The last kernel liborion enqueued per stream (orion_internal.h).
static std::mutex g_tag_mu;
static std::unordered_map<CUstream, const void *> g_stream_tag;

void orion::note_stream_launch(CUstream s, const void *tag)
{
    std::lock_guard<std::mutex> lk(g_tag_mu);
    g_stream_tag[s] = tag;
}
const void *orion::last_stream_tag(CUstream s)
{
    std::lock_guard<std::mutex> lk(g_tag_mu);
    auto it = g_stream_tag.find(s);
    return it == g_stream_tag.end() ? nullptr : it->second;
}

namespace {

// The ROI of a fused-statistics SRAD launch: fparam[1..4] = r1, r2, c1, c2 (inclusive, exact
// integers), inside the grid, and few enough (strip, block) slots for the statistics area.
orion_status check_srad_roi(int W, int H, const float *f, int strip_rows)
{
    int v[4];
    for (int i = 0; i < 4; ++i) {
        v[i] = (int)f[i];
        if ((float)v[i] != f[i]) return fail(ORION_E_INVALID, "srad ROI: fparam[1..4] must be integers");
    }
    if (v[0] < 0 || v[0] > v[1] || v[1] >= H || v[2] < 0 || v[2] > v[3] || v[3] >= W)
        return fail(ORION_E_INVALID, "srad ROI outside the grid");
    const int slots = (v[1] / strip_rows - v[0] / strip_rows + 1) * (v[3] / 120 - v[2] / 120 + 1);
    if (slots > ORION_SRAD_STAT_SLOTS) return fail(ORION_E_INVALID, "srad ROI spans too many statistics slots");
    return ORION_OK;
}

int warps_of(const orion_device_limits &d, int T) { return (T + d.warp_size - 1) / d.warp_size; }

// Translate the public argument block into the kernel's parameter block, checking that
// the source slab holds every row the kernel reaches (clamped to the image).
orion_status make_kargs(const KernelDef &def, const orion_args *a, orion_kargs *k)
{
    std::memset(k, 0, sizeof *k);          // an empty launch still hands back a defined block
    if (!a) return fail(ORION_E_INVALID, "orion_launch: NULL args");
    if (a->width <= 0 || a->height <= 0 || a->row_begin < 0 || a->row_end > a->height || a->row_begin > a->row_end)
        return fail(ORION_E_INVALID, "orion_launch: bad image geometry");
    if (a->row_begin == a->row_end) return ORION_OK;
    if (!a->src || !a->dst || ((def.kind == K_STENCIL || (def.kind == K_SRAD && !def.srad_stats)) && !a->aux))
        return fail(ORION_E_INVALID, "orion_launch: NULL buffer");
    if (def.srad_stats) {
        if (a->row_begin != 0 || a->row_end != a->height || a->src_row_begin != 0 || a->dst_row_begin != 0)
            return fail(ORION_E_INVALID, std::string("orion_launch: ") + def.id + ": whole grids only");
        ORION_TRY(check_srad_roi(a->width, a->height, a->fparam + 1, def.tile_h / 8));
    }
    const int need_lo = std::max(0, a->row_begin - def.halo);
    const int need_hi = std::min(a->height, a->row_end + def.halo);
    if (a->src_row_begin > need_lo || a->src_row_end < need_hi)
        return fail(ORION_E_INVALID, "orion_launch: src rows do not cover the halo of the output rows");
    if (a->dst_row_begin > a->row_begin) return fail(ORION_E_INVALID, "orion_launch: dst_row_begin > row_begin");
    if (def.width_align > 1 && a->width % def.width_align)
        return fail(ORION_E_INVALID, std::string("orion_launch: ") + def.id + " needs width % " +
                                         std::to_string(def.width_align) + " == 0");
    if (a->n_fanout < 0 || a->n_fanout > 8 || (a->n_fanout > 0 && !def.fanout))
        return fail(ORION_E_INVALID, std::string("orion_launch: ") + def.id + ": bad n_fanout");
    if (def.kind == K_STENCIL) {
        // the halo exchange: exactly (upper, lower) neighbour buffers, NULL at the grid's edge
        if (a->n_fanout != 0 && a->n_fanout != 2)
            return fail(ORION_E_INVALID, std::string("orion_launch: ") + def.id + ": n_fanout must be 0 or 2");
    } else {
        for (int f = 0; f < a->n_fanout; ++f)
            if (!a->fanout[f]) return fail(ORION_E_INVALID, "orion_launch: NULL fanout buffer");
    }
    for (int f = 0; f < a->n_fanout; ++f) k->fan[f] = a->fanout[f];
    k->nfan = a->n_fanout;
    if (a->flags & ~ORION_ARGS_INDEPENDENT) return fail(ORION_E_INVALID, "orion_launch: unknown flags");
    if ((a->flags & ORION_ARGS_INDEPENDENT) && (def.kind == K_STENCIL || def.kind == K_SRAD))
        return fail(ORION_E_INVALID, std::string("orion_launch: ") + def.id +
                                         ": a stencil launch reads its predecessor's output (not independent)");
    k->nowait = (a->flags & ORION_ARGS_INDEPENDENT) ? 1 : 0;
    k->batch = 1;
    if (a->batch < 0 || a->batch > 65535) return fail(ORION_E_INVALID, "orion_launch: batch out of range");
    if (a->batch > 1) {
        if (def.kind == K_STENCIL || def.kind == K_SRAD)
            return fail(ORION_E_INVALID, std::string("orion_launch: ") + def.id + ": batches are for the denoisers");
        if (a->row_begin != 0 || a->row_end != a->height || a->src_row_begin != 0 || a->src_row_end != a->height ||
            a->dst_row_begin != 0 || a->n_fanout || a->chain)
            return fail(ORION_E_INVALID, "orion_launch: a batch holds whole frames (no bands, fan-out or chain)");
        k->batch = a->batch;
    }
    if (a->chain) {
        const orion_chain *c = a->chain;
        if (!def.chain || c->def != &def)
            return fail(ORION_E_INVALID, std::string("orion_launch: ") + def.id + ": chain of another kernel family");
        if (a->width != c->width || a->height != c->height || a->row_begin != 0 || a->row_end != a->height ||
            a->src_row_begin != 0 || a->src_row_end != a->height || a->dst_row_begin != 0)
            return fail(ORION_E_INVALID, "orion_launch: a chained launch covers the chain's whole grid");
        if (a->flags || a->n_fanout)
            return fail(ORION_E_INVALID, "orion_launch: a chained launch takes no flags / fan-out");
        if (t_capturing)
            return fail(ORION_E_INVALID, "orion_launch: chained launches cannot be captured (epochs advance per launch)");
    }
    k->src = a->src;
    k->dst = a->dst;
    k->aux = a->aux;
    k->width = a->width;
    k->height = a->height;
    k->row_begin = a->row_begin;
    k->row_end = a->row_end;
    k->src_row_begin = a->src_row_begin;
    k->src_row_end = a->src_row_end;
    k->dst_row_begin = a->dst_row_begin;
    if (def.kind == K_STENCIL || def.kind == K_SRAD) {
        for (int i = 0; i < 8; ++i) k->fparam[i] = a->fparam[i];
    } else {
        // SDK parameters -> kernel form: w = 2^(d * (-Noise log2 e) + geo); count threshold
        // "cnt/A > lthr" on an integer count == cnt >= floor(lthr*A) + 1.
        const double noise = a->fparam[0];
        if (!(noise >= 0.0)) return fail(ORION_E_INVALID, "orion_launch: Noise must be >= 0");
        k->fparam[0] = (float)(-noise * 1.4426950408889634);
        k->fparam[1] = a->fparam[1];
        k->fparam[2] = a->fparam[2];
        // the weight threshold as an exponent (w = 2^e, flushed to 0 below 2^-126)
        const double wt = a->fparam[2];
        k->fparam[3] = wt > 0.0 ? (float)std::log2(wt) : (wt == 0.0 ? -126.0f : -INFINITY);
        k->iparam0 = (int)std::floor((double)a->fparam[3] * 49.0) + 1;
    }
    return ORION_OK;
}

// Launches use programmatic stream serialization (PDL) unless ORION_PDL=0, and never while a
// graph is being captured.  Measured A/B on one box (same library, ORION_PDL=0 vs 1): C2
// 0.2217 -> 0.2197 ms, SRAD 0.1044 -> 0.1029 ms, C3 0.1571 -> 0.1564 ms per launch.
// -1: not yet read from ORION_PDL; orion_set_pdl() overrides it at run time.
static std::atomic<int> g_pdl{-1};

static bool pdl_enabled()
{
    int on = g_pdl.load();
    if (on < 0) {
        const char *e = std::getenv("ORION_PDL");
        int want = (e && e[0] == '0') ? 0 : 1;
        g_pdl.compare_exchange_strong(on, want);
        on = g_pdl.load();
    }
    return on && (!t_capturing || t_capture_pdl);
}

static int pdl_enabled_setting()
{
    const bool cap = t_capturing;
    t_capturing = false;
    const int on = pdl_enabled() ? 1 : 0;
    t_capturing = cap;
    return on;
}

// Programmatic dependent launch when enabled: this grid may be scheduled while the previous
// kernel of the stream drains; every kernel waits (griddepcontrol.wait, kernels/common.cuh and
// orion_srad_stats) for its predecessor's completion before touching memory, so results are
// unchanged.
static orion_status launch_maybe_pdl(CUfunction fn, unsigned gx, unsigned gy, unsigned gz, unsigned bx, unsigned by,
                                     unsigned smem, CUstream s, void **params, const void *tag = nullptr)
{
    note_stream_launch(s, tag);
    if (!pdl_enabled()) {
        ORION_CU(drv().cuLaunchKernel(fn, gx, gy, gz, bx, by, 1, smem, s, params, nullptr));
        return ORION_OK;
    }
    CUlaunchAttribute attr;
    std::memset(&attr, 0, sizeof attr);
    attr.id = CU_LAUNCH_ATTRIBUTE_PROGRAMMATIC_STREAM_SERIALIZATION;
    attr.value.programmaticStreamSerializationAllowed = 1;
    CUlaunchConfig cfg;
    std::memset(&cfg, 0, sizeof cfg);
    cfg.gridDimX = gx;
    cfg.gridDimY = gy;
    cfg.gridDimZ = gz;
    cfg.blockDimX = bx;
    cfg.blockDimY = by;
    cfg.blockDimZ = 1;
    cfg.sharedMemBytes = smem;
    cfg.hStream = s;
    cfg.attrs = &attr;
    cfg.numAttrs = 1;
    ORION_CU(drv().cuLaunchKernelEx(&cfg, fn, params, nullptr));
    return ORION_OK;
}


orion_status launch_fn(const KernelDef &def, CUfunction fn, int dyn_bytes, const orion_kargs &k, CUstream s,
                       const void *tag = nullptr)
{
    const int rows = k.row_end - k.row_begin;
    if (rows <= 0) return ORION_OK;
    const unsigned gx = (unsigned)((k.width + def.tile_w - 1) / def.tile_w);
    const unsigned gy = (unsigned)((rows + def.tile_h - 1) / def.tile_h);
    void *params[] = {const_cast<orion_kargs *>(&k)};
    const unsigned gz = (unsigned)(k.batch > 1 ? k.batch : 1);    // frames of a batched launch
    ORION_TRY(launch_maybe_pdl(fn, gx, gy, gz, (unsigned)def.bx, (unsigned)def.by, (unsigned)dyn_bytes, s, params, tag));
    g_launches.fetch_add(1);
    return ORION_OK;
}

// Device scratch of the residency probe: 1024 live counters + 1024 maxima (per %smid).
struct ProbeBuffer {
    CUdeviceptr p = 0;
    orion_status alloc()
    {
        if (drv().cuMemAlloc(&p, 2048 * sizeof(unsigned)) != CUDA_SUCCESS) {
            p = 0;
            return fail(ORION_E_CUDA, "cuMemAlloc (residency probe)");
        }
        return ORION_OK;
    }
    ~ProbeBuffer()
    {
        if (p) drv().cuMemFree(p);
    }
};

// Launch `fn` as a residency probe (kargs.probe set: every CTA only counts its SM's resident
// CTAs, then holds for 20 us) over sm_count x 32 CTAs, and return the largest number of CTAs
// ever resident together on one SM.
orion_status measure_residency(const orion_variants &v, const KernelDef &def, CUfunction fn, int dyn_bytes,
                               const ProbeBuffer &buf, int *out)
{
    const Driver &D = drv();
    ORION_CU(D.cuMemsetD32(buf.p, 0u, 2048));
    orion_kargs k;
    std::memset(&k, 0, sizeof k);
    k.probe = reinterpret_cast<unsigned *>(buf.p);
    void *params[] = {&k};
    const unsigned grid = (unsigned)(v.dev.sm_count * v.dev.max_blocks_per_sm);
    note_stream_launch(nullptr, nullptr);
    ORION_CU(D.cuLaunchKernel(fn, grid, 1, 1, (unsigned)def.bx, (unsigned)def.by, 1, (unsigned)dyn_bytes, nullptr,
                              params, nullptr));
    ORION_CU(D.cuCtxSynchronize());
    unsigned host[1024];
    ORION_CU(D.cuMemcpyDtoH(host, buf.p + 1024 * sizeof(unsigned), sizeof host));
    unsigned m = 0;
    for (unsigned x : host) m = std::max(m, x);
    *out = (int)m;
    return ORION_OK;
}

}  // namespace

extern "C" {

orion_status orion_build_variants(int device, const char *kernel_id, int block_threads, const orion_level *levels,
                                  int n, orion_variants **out)
{
    if (!out || !levels || n <= 0) return fail(ORION_E_INVALID, "orion_build_variants: bad argument");
    *out = nullptr;
    const KernelDef *def = find_kernel(kernel_id, block_threads);
    if (!def) return fail(ORION_E_INVALID, std::string("unknown kernel ") + (kernel_id ? kernel_id : "(null)"));
    ORION_TRY(ensure_context(device));
    auto v = new orion_variants();
    std::unique_ptr<orion_variants, void (*)(orion_variants *)> guard(v, orion_variants_destroy);
    v->device = device;
    v->def = def;
    ORION_TRY(orion_query_limits(device, &v->dev));
    ORION_TRY(orion_kernel_probe(kernel_id, def->threads, &v->res));
    const Driver &D = drv();
    const int T = def->threads;
    const int need = def->dyn_need();
    ProbeBuffer probe;
    ORION_TRY(probe.alloc());
    for (int i = 0; i < n; ++i) {
        const orion_level &L = levels[i];
        if (L.ctas_per_sm < 1 || L.reg_cap < 0 || L.reg_cap > 255)
            return fail(ORION_E_INVALID, "orion_build_variants: bad level");
        orion_variants::Var var;
        var.planned = L;
        ORION_TRY(compile_variant(*def, L.reg_cap, &var.cv));
        ORION_CU(D.cuModuleLoadData(&var.mod, var.cv->cubin.data()));
        v->vars.push_back(var);   // owns the module from here on (destroy unloads it)
        orion_variants::Var &w = v->vars.back();
        ORION_CU(D.cuModuleGetFunction(&w.fn, w.mod, def->entry));
        int static_smem = 0;
        ORION_CU(D.cuFuncGetAttribute(&w.regs, CU_FUNC_ATTRIBUTE_NUM_REGS, w.fn));
        ORION_CU(D.cuFuncGetAttribute(&w.local_bytes, CU_FUNC_ATTRIBUTE_LOCAL_SIZE_BYTES, w.fn));
        ORION_CU(D.cuFuncGetAttribute(&static_smem, CU_FUNC_ATTRIBUTE_SHARED_SIZE_BYTES, w.fn));
        // Realise level k: the planned carveout first, then every larger configuration.  A
        // candidate is accepted when both the driver's occupancy API AND the measured
        // residency (a probe launch of this very function, orion_probe in common.cuh) give k:
        // the driver treats the carveout preference as a hint and may run a padded launch in a
        // larger configuration than requested (measured on B200: an 8 KB preference runs in
        // 16 or 64 KB), which the occupancy API does not model.
        std::vector<int> pcts{level_carveout_pct(v->dev, L)};
        {
            int nc = 0;
            const int *kb = carveout_configs_kb(&nc);
            for (int c = 0; c < nc; ++c)
                if (kb[c] > std::max(L.carveout_kb, 0) && (long long)kb[c] * 1024 <= v->dev.smem_per_sm)
                    pcts.push_back(kb[c] * 1024 >= v->dev.smem_per_sm ? 100 : carveout_pct_for_kb(v->dev, kb[c]));
        }
        int pct = -1, pad = -1, api = 0, measured = 0;
        bool ok = false;
        std::string tried;
        for (int cand : pcts) {
            pct = cand;
            pad = pad_for_level(v->dev, T, w.regs, static_smem, need, L.ctas_per_sm, pct);
            if (pad > 0 && pct < 0) {   // padding needed at the actual register count: pin the maximum
                pct = 100;
                pad = pad_for_level(v->dev, T, w.regs, static_smem, need, L.ctas_per_sm, pct);
            }
            if (pad < 0) continue;
            w.dyn_bytes = need + pad;
            ORION_CU(D.cuFuncSetAttribute(w.fn, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, w.dyn_bytes));
            if (pct >= 0) ORION_CU(D.cuFuncSetAttribute(w.fn, CU_FUNC_ATTRIBUTE_PREFERRED_SHARED_MEMORY_CARVEOUT, pct));
            ORION_CU(D.cuOccupancyMaxActiveBlocksPerMultiprocessor(&api, w.fn, T, (size_t)w.dyn_bytes));
            if (api != L.ctas_per_sm) {
                tried += " pct " + std::to_string(pct) + ": api " + std::to_string(api) + ";";
                continue;
            }
            ORION_TRY(measure_residency(*v, *def, w.fn, w.dyn_bytes, probe, &measured));
            tried += " pct " + std::to_string(pct) + ": measured " + std::to_string(measured) + ";";
            if (measured == L.ctas_per_sm) {
                ok = true;
                break;
            }
        }
        if (!ok)
            return fail(ORION_E_OCCUPANCY_MISMATCH, std::string(def->entry) + ": level " +
                                                        std::to_string(L.ctas_per_sm) + " not realisable at " +
                                                        std::to_string(w.regs) + " registers (" + tried + ")");
        w.carveout_pct = pct;
        w.verified = measured;
        w.realised = L;
        w.realised.smem_pad_bytes = pad;
        int limiter = 0;
        ctas_per_sm(v->dev, T, w.regs, static_smem, w.dyn_bytes, pct, &limiter);
        w.realised.limiter = limiter;
        w.realised.carveout_kb = pct < 0 ? 0 : carveout_pref_bytes(v->dev, pct) / 1024;
        w.realised.warps_per_sm = L.ctas_per_sm * warps_of(v->dev, T);
        w.realised.occupancy_permille = w.realised.warps_per_sm * 1000 / (v->dev.max_threads_per_sm / v->dev.warp_size);
    }
    *out = guard.release();
    return ORION_OK;
}

void orion_variants_destroy(orion_variants *v)
{
    if (!v) return;
    if (drv().ok)
        for (auto &w : v->vars)
            if (w.mod) drv().cuModuleUnload(w.mod);
    delete v;
}

orion_status orion_variants_count(const orion_variants *v, int *n)
{
    if (!v || !n) return fail(ORION_E_INVALID, "orion_variants_count: NULL");
    *n = (int)v->vars.size();
    return ORION_OK;
}

orion_status orion_variant_level(const orion_variants *v, int i, orion_level *out)
{
    if (!v || !out || i < 0 || i >= (int)v->vars.size()) return fail(ORION_E_INVALID, "orion_variant_level");
    *out = v->vars[i].realised;
    return ORION_OK;
}

orion_status orion_variant_info(const orion_variants *v, int i, int *regs, int *spill_st, int *spill_ld,
                                int *local_bytes, int *verified)
{
    if (!v || i < 0 || i >= (int)v->vars.size()) return fail(ORION_E_INVALID, "orion_variant_info");
    const auto &w = v->vars[i];
    if (regs) *regs = w.regs;
    if (spill_st) *spill_st = w.cv->spill_store;
    if (spill_ld) *spill_ld = w.cv->spill_load;
    if (local_bytes) *local_bytes = w.local_bytes;
    if (verified) *verified = w.verified;
    return ORION_OK;
}

orion_status orion_variants_resources(const orion_variants *v, orion_kernel_resources *out)
{
    if (!v || !out) return fail(ORION_E_INVALID, "orion_variants_resources: NULL");
    *out = v->res;
    return ORION_OK;
}

orion_status orion_launch(orion_variants *v, int i, const orion_args *a, void *stream)
{
    if (!v || i < 0 || i >= (int)v->vars.size()) return fail(ORION_E_INVALID, "orion_launch: bad variant");
    orion_kargs k;
    ORION_TRY(make_kargs(*v->def, a, &k));
    if (a->row_begin == a->row_end) return ORION_OK;
    ORION_TRY(ensure_context(v->device));
    const auto &w = v->vars[i];
    orion_chain *c = a->chain;
    if (!c) return launch_fn(*v->def, w.fn, w.dyn_bytes, k, (CUstream)stream);
    if (c->device != v->device) return fail(ORION_E_INVALID, "orion_launch: chain of another device");
    if (c->stream_set && c->stream != (CUstream)stream)
        return fail(ORION_E_INVALID, "orion_launch: a chain's launches go to one stream");
    k.chain = (unsigned *)c->flags;
    k.chain_epoch = c->epoch + 1;
    // tile-level waits replace the grid-wide wait only right behind this chain's previous launch;
    // behind any other kernel of liborion (or the chain's first launch) the launch waits as usual
    k.nowait = (c->epoch > 0 && last_stream_tag((CUstream)stream) == (const void *)c) ? 1 : 0;
    k.dep_late = v->def->srad_stats ? 1 : 0;
    ORION_TRY(launch_fn(*v->def, w.fn, w.dyn_bytes, k, (CUstream)stream, c));
    c->epoch += 1;
    c->stream = (CUstream)stream;
    c->stream_set = true;
    return ORION_OK;
}

orion_status orion_chain_create(const orion_variants *v, int width, int height, orion_chain **out)
{
    if (!v || !out || width <= 0 || height <= 0) return fail(ORION_E_INVALID, "orion_chain_create: bad argument");
    *out = nullptr;
    if (!v->def->chain)
        return fail(ORION_E_INVALID, std::string("orion_chain_create: ") + v->def->id + " does not take a chain");
    ORION_TRY(ensure_context(v->device));
    std::unique_ptr<orion_chain> c(new orion_chain());
    c->device = v->device;
    c->def = v->def;
    c->width = width;
    c->height = height;
    c->gx = (width + v->def->tile_w - 1) / v->def->tile_w;
    c->gy = (height + v->def->tile_h - 1) / v->def->tile_h;
    const size_t bytes = (size_t)c->gx * (size_t)c->gy * sizeof(unsigned);
    if (drv().cuMemAlloc(&c->flags, bytes) != CUDA_SUCCESS) return fail(ORION_E_CUDA, "cuMemAlloc (chain flags)");
    if (drv().cuMemsetD32(c->flags, 0u, bytes / sizeof(unsigned)) != CUDA_SUCCESS) {
        drv().cuMemFree(c->flags);
        return fail(ORION_E_CUDA, "cuMemsetD32 (chain flags)");
    }
    *out = c.release();
    return ORION_OK;
}

void orion_chain_destroy(orion_chain *c)
{
    if (!c) return;
    if (drv().ok && c->flags && ensure_context(c->device) == ORION_OK) drv().cuMemFree(c->flags);
    delete c;
}

orion_status orion_chain_info(const orion_chain *c, unsigned *epoch, int *tiles_x, int *tiles_y)
{
    if (!c) return fail(ORION_E_INVALID, "orion_chain_info: NULL");
    if (epoch) *epoch = c->epoch;
    if (tiles_x) *tiles_x = c->gx;
    if (tiles_y) *tiles_y = c->gy;
    return ORION_OK;
}

orion_status orion_default_params(const char *kernel_id, float *fparam, int n)
{
    if (!kernel_id || !fparam || n < 8) return fail(ORION_E_INVALID, "orion_default_params: bad argument");
    const KernelDef *def = find_kernel(kernel_id, 0);
    if (!def) return fail(ORION_E_INVALID, std::string("orion_default_params: unknown kernel ") + kernel_id);
    for (int i = 0; i < n; ++i) fparam[i] = 0.0f;
    switch (def->kind) {
    case K_KNN:      // CUDA-SDK imageDenoising KNN (reading R-O2): Noise = 1/h^2, h = 0.32
        fparam[0] = (float)(1.0 / (0.32 * 0.32));
        fparam[1] = 0.2f;          // lerpC
        fparam[2] = 0.02f;         // weight threshold
        fparam[3] = 0.79f;         // lerp threshold on cnt / 49
        break;
    case K_NLM:      // CUDA-SDK imageDenoising NLM (reading R-O2): h = 1.45
        fparam[0] = (float)(1.0 / (1.45 * 1.45));
        fparam[1] = 0.2f;
        fparam[2] = 0.10f;
        fparam[3] = 0.10f;
        break;
    case K_STENCIL: {  // Rodinia hotspot at the 512-grid cell size for every N (readings R-O3, R-A15)
        const double cell = 0.016 / 512.0;       // 16 mm chip / 512 cells = 31.25 um
        const double t_chip = 0.0005, k_si = 100.0, spec_heat_si = 1.75e6, factor_chip = 0.5;
        const double max_pd = 3.0e6, precision = 0.001, amb = 80.0;
        const double cap = factor_chip * spec_heat_si * t_chip * cell * cell;
        const double r_x = cell / (2.0 * k_si * t_chip * cell);
        const double r_y = cell / (2.0 * k_si * t_chip * cell);
        const double r_z = t_chip / (k_si * cell * cell);
        const double step = precision / (max_pd / (factor_chip * t_chip * spec_heat_si));
        fparam[0] = (float)(step / cap);         // sdc = step / Cap
        fparam[1] = (float)(1.0 / r_x);          // rx = 1 / Rx
        fparam[2] = (float)(1.0 / r_y);          // ry = 1 / Ry
        fparam[3] = (float)(1.0 / r_z);          // rz = 1 / Rz
        fparam[4] = (float)amb;
        break;
    }
    case K_SRAD:     // Rodinia srad_v2 (reading R-SRAD): lambda = 0.5
        fparam[0] = 0.5f;
        break;
    default:
        return fail(ORION_E_INVALID, "orion_default_params: kernel without method parameters");
    }
    return ORION_OK;
}

orion_status orion_set_pdl(int on, int *previous)
{
    if (on != 0 && on != 1) return fail(ORION_E_INVALID, "orion_set_pdl: on must be 0 or 1");
    const int was = pdl_enabled_setting();
    g_pdl.store(on);
    if (previous) *previous = was;
    return ORION_OK;
}

orion_status orion_sweep(orion_variants *v, const orion_args *a, void *stream, int rounds, float *ms_median)
{
    if (!v || !a || rounds <= 0 || !ms_median) return fail(ORION_E_INVALID, "orion_sweep: bad argument");
    if (a->chain) return fail(ORION_E_INVALID, "orion_sweep: repeats one launch -- time it without a chain");
    orion_kargs k;
    ORION_TRY(make_kargs(*v->def, a, &k));
    if (a->row_begin == a->row_end) {     // nothing to time: an empty launch is a no-op at every level
        for (size_t i = 0; i < v->vars.size(); ++i) ms_median[i] = 0.0f;
        return ORION_OK;
    }
    ORION_TRY(ensure_context(v->device));
    const Driver &D = drv();
    const int n = (int)v->vars.size();
    CUstream s = (CUstream)stream;
    std::vector<CUevent> ev((size_t)2 * n * rounds, nullptr);
    orion_status st = ORION_OK;
    for (auto &e : ev)
        if (D.cuEventCreate(&e, CU_EVENT_DEFAULT) != CUDA_SUCCESS) {
            st = fail(ORION_E_CUDA, "cuEventCreate");
            break;
        }
    // warm every variant once (module lazy loading, instruction cache) and time that launch:
    // a level whose launch is shorter than kMinSampleMs is timed over a batch of back-to-back
    // launches per sample (per-launch ms = batch ms / batch), so event overhead and launch
    // jitter do not decide between microsecond-scale levels
    constexpr float kMinSampleMs = 0.2f;
    std::vector<int> batch((size_t)n, 1);
    for (int i = 0; i < n && st == ORION_OK; ++i) {
        float w = 0.0f;
        if (D.cuEventRecord(ev[0], s) != CUDA_SUCCESS) st = fail(ORION_E_CUDA, "cuEventRecord");
        if (st == ORION_OK) st = launch_fn(*v->def, v->vars[i].fn, v->vars[i].dyn_bytes, k, s);
        if (st == ORION_OK && (D.cuEventRecord(ev[1], s) != CUDA_SUCCESS || D.cuEventSynchronize(ev[1]) != CUDA_SUCCESS ||
                               D.cuEventElapsedTime(&w, ev[0], ev[1]) != CUDA_SUCCESS))
            st = fail(ORION_E_CUDA, "sweep warm-up timing");
        if (st == ORION_OK && w > 0.0f && w < kMinSampleMs)
            batch[(size_t)i] = std::min(64, (int)std::ceil(kMinSampleMs / w));
    }
    if (st == ORION_OK) {
        for (int r = 0; r < rounds && st == ORION_OK; ++r)
            for (int q = 0; q < n && st == ORION_OK; ++q) {
                const int i = (q + r) % n;   // rotate the start so no level is always first
                const size_t e = (size_t)2 * (r * n + i);
                if (D.cuEventRecord(ev[e], s) != CUDA_SUCCESS) st = fail(ORION_E_CUDA, "cuEventRecord");
                for (int b = 0; b < batch[(size_t)i] && st == ORION_OK; ++b)
                    st = launch_fn(*v->def, v->vars[i].fn, v->vars[i].dyn_bytes, k, s);
                if (st == ORION_OK && D.cuEventRecord(ev[e + 1], s) != CUDA_SUCCESS)
                    st = fail(ORION_E_CUDA, "cuEventRecord");
            }
        if (st == ORION_OK && D.cuStreamSynchronize(s) != CUDA_SUCCESS) st = fail(ORION_E_CUDA, "cuStreamSynchronize");
        if (st == ORION_OK) {
            std::vector<float> t(rounds);
            for (int i = 0; i < n && st == ORION_OK; ++i) {
                for (int r = 0; r < rounds; ++r) {
                    const size_t e = (size_t)2 * (r * n + i);
                    if (D.cuEventElapsedTime(&t[r], ev[e], ev[e + 1]) != CUDA_SUCCESS) {
                        st = fail(ORION_E_CUDA, "cuEventElapsedTime");
                        break;
                    }
                }
                std::sort(t.begin(), t.end());
                ms_median[i] = ((rounds % 2) ? t[rounds / 2] : 0.5f * (t[rounds / 2 - 1] + t[rounds / 2])) /
                               (float)batch[(size_t)i];
            }
        }
    }
    for (auto &e : ev)
        if (e) D.cuEventDestroy(e);
    return st;
}

// ---- synthetic inputs -------------------------------------------------------------------
// The device twin of synth/ (a separate implementation of the same counter-based
// generator; no method arithmetic).  Box geometry is drawn here on the host.
struct orion_boxes { int x0[12], y0[12], w[12], h[12]; float r[12], g[12], b[12]; };

static uint64_t splitmix64_host(uint64_t x)
{
    uint64_t z = x + 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

orion_status orion_generate_rgba(int device, void *dst, int W, int H, int row_begin, int row_end, unsigned seed,
                                 float sigma, void *stream)
{
    if (!dst || W <= 0 || H <= 0 || row_begin < 0 || row_end > H || row_begin > row_end || seed >= (1u << 24))
        return fail(ORION_E_INVALID, "orion_generate_rgba: bad argument");
    if (row_begin == row_end) return ORION_OK;
    CUmodule m;
    ORION_TRY(load_aux_module(device, "gen", &m));
    CUfunction f;
    ORION_CU(drv().cuModuleGetFunction(&f, m, "orion_gen_rgba"));
    orion_boxes bx;
    for (int b = 0; b < 12; ++b) {
        uint64_t h[5];
        for (int k = 0; k < 5; ++k)
            h[k] = splitmix64_host(((uint64_t)seed << 40) | (1ull << 39) | (uint64_t)(b * 8 + k));
        bx.x0[b] = (int)(h[0] % (uint64_t)W);
        bx.y0[b] = (int)(h[1] % (uint64_t)H);
        bx.w[b] = 1 + (int)(h[2] % (uint64_t)std::max(1, W / 4));
        bx.h[b] = 1 + (int)(h[3] % (uint64_t)std::max(1, H / 4));
        bx.r[b] = (float)(((h[4] >> 0) % 820 + 102) / 1024.0);
        bx.g[b] = (float)(((h[4] >> 16) % 820 + 102) / 1024.0);
        bx.b[b] = (float)(((h[4] >> 32) % 820 + 102) / 1024.0);
    }
    const float s = (float)(std::sqrt(3.0) * (double)sigma);
    unsigned long long sd = seed;
    void *params[] = {&dst, &W, &H, &row_begin, &row_end, &sd, (void *)&s, &bx};
    note_stream_launch((CUstream)stream, nullptr);
    ORION_CU(drv().cuLaunchKernel(f, (unsigned)((W + 255) / 256), (unsigned)(row_end - row_begin), 1, 256, 1, 1, 0,
                                  (CUstream)stream, params, nullptr));
    g_launches.fetch_add(1);
    return ORION_OK;
}

orion_status orion_generate_thermal(int device, void *t0, void *pw, int W, int H, unsigned seed, void *stream)
{
    if (!t0 || !pw || W <= 0 || H <= 0 || seed >= (1u << 24))
        return fail(ORION_E_INVALID, "orion_generate_thermal: bad argument");
    CUmodule m;
    ORION_TRY(load_aux_module(device, "gen", &m));
    CUfunction f;
    ORION_CU(drv().cuModuleGetFunction(&f, m, "orion_gen_thermal"));
    unsigned long long sd = seed;
    void *params[] = {&t0, &pw, &W, &H, &sd};
    note_stream_launch((CUstream)stream, nullptr);
    ORION_CU(drv().cuLaunchKernel(f, (unsigned)((W + 255) / 256), (unsigned)H, 1, 256, 1, 1, 0, (CUstream)stream,
                                  params, nullptr));
    g_launches.fetch_add(1);
    return ORION_OK;
}

orion_status orion_flush_l2(int device, void *buf, long long bytes, void *stream)
{
    if (!buf || bytes < 16) return fail(ORION_E_INVALID, "orion_flush_l2: bad argument");
    CUmodule m;
    ORION_TRY(load_aux_module(device, "gen", &m));
    CUfunction f;
    ORION_CU(drv().cuModuleGetFunction(&f, m, "orion_l2_flush"));
    size_t n = (size_t)(bytes / 16);
    float val = 0.0f;
    void *params[] = {&buf, &n, &val};
    note_stream_launch((CUstream)stream, nullptr);
    ORION_CU(drv().cuLaunchKernel(f, 148 * 8, 1, 1, 256, 1, 1, 0, (CUstream)stream, params, nullptr));
    g_launches.fetch_add(1);
    return ORION_OK;
}

}  // extern "C"

extern "C" orion_status orion_srad_stats_init(int device, void *J, int width, int height, int r1, int r2, int c1,
                                              int c2, void *stream)
{
    if (!J || width <= 0 || height <= 0 || width % 4) return fail(ORION_E_INVALID, "orion_srad_stats_init: bad argument");
    const KernelDef *def = find_kernel("srad_f32hs", 0);
    orion_kargs k;
    std::memset(&k, 0, sizeof k);
    k.src = J;
    k.width = width;
    k.height = height;
    k.row_end = height;
    k.src_row_end = height;
    k.fparam[1] = (float)r1;
    k.fparam[2] = (float)r2;
    k.fparam[3] = (float)c1;
    k.fparam[4] = (float)c2;
    ORION_TRY(check_srad_roi(width, height, k.fparam + 1, def->tile_h / 8));
    const int rows = def->tile_h / 8;
    const int slots = (r2 / rows - r1 / rows + 1) * (c2 / 120 - c1 / 120 + 1);
    CUmodule m;
    ORION_TRY(load_aux_module(device, "srad", &m));
    CUfunction f;
    ORION_CU(drv().cuModuleGetFunction(&f, m, "orion_srad_stats_init"));
    void *params[] = {&k};
    ORION_TRY(launch_maybe_pdl(f, (unsigned)slots, 1, 1, 32, 1, 0, (CUstream)stream, params));
    g_launches.fetch_add(1);
    return ORION_OK;
}

extern "C" orion_status orion_srad_roi_stats(int device, const void *J, int width, int height, int r1, int r2, int c1,
                                             int c2, void *q0, void *stream)
{
    if (!J || !q0 || width <= 0 || height <= 0 || r1 < 0 || c1 < 0 || r2 < r1 || c2 < c1 || r2 >= height ||
        c2 >= width)
        return fail(ORION_E_INVALID, "orion_srad_roi_stats: bad argument");
    CUmodule m;
    ORION_TRY(load_aux_module(device, "srad", &m));
    CUfunction f;
    ORION_CU(drv().cuModuleGetFunction(&f, m, "orion_srad_stats"));
    void *params[] = {&J, &width, &r1, &r2, &c1, &c2, &q0};
    ORION_TRY(launch_maybe_pdl(f, 1, 1, 1, 1024, 1, 0, (CUstream)stream, params));
    g_launches.fetch_add(1);
    return ORION_OK;
}
