// tuner.cpp -- Orion's two-level selection (Fig. 3):
//   level 1, compile time: Fig. 8's occupancy update algorithm prunes the levels to a
//            candidate ladder (P:L583-P:L603, P:L645-P:L649);
//   level 2, run time:     Fig. 9's dynamic occupancy selection walks that ladder across
//            the application's iterations and settles on a final kernel (P:L605-P:L643,
//            P:L651-P:L653, P:L687-P:L689).
//
// Readings: MAXLIVE = the natural register count (R-A5); conservative = the
// first register-cap rung above the original (R-A6); canTune = iterations >= |ladder|+2
// (R-A7); "Slowdown > .02" is measured against the best so far (R-A3); the final kernel
// is the fastest measured (ties -> lower occupancy, Principle 2 P:L181-P:L183) or, in
// LOWEST_WITHIN_TOL mode, the lowest occupancy within slowdown_tol of the best (R-A4).
#include <algorithm>
#include <map>
#include <memory>

#include "orion_internal.h"

using namespace orion;

namespace {

struct Fig9 {
    orion_tuner_cfg cfg{};
    std::vector<int> ks;        // CTAs/SM of every level (index = level idx)
    int direction = ORION_DIR_INCREASING;
    std::vector<int> ladder, other;
    int cur = -1;               // ladder position last run (-1: nothing run yet)
    float best = 0.0f;
    int final_idx = -1, final_iter = -1;
    bool switched = false;
    int iter = 0;
    std::map<int, float> tried; // level idx -> measured ms

    // Fig. 8 (canTune branch): ladders from the level list and MAXLIVE.
    void prune(const orion_level *lv, int n, int natural_regs)
    {
        ks.resize(n);
        // the original: the most CTAs the natural register count admits; a rung
        // of the register ladder: the most CTAs a given register cap admits
        std::map<int, int> top_of_cap;   // reg_cap -> level index with the largest k
        for (int i = 0; i < n; ++i) {
            ks[i] = lv[i].ctas_per_sm;
            auto it = top_of_cap.find(lv[i].reg_cap);
            if (it == top_of_cap.end() || ks[i] > ks[it->second]) top_of_cap[lv[i].reg_cap] = i;
        }
        const int orig = top_of_cap.at(0);
        const int k0 = ks[orig];
        std::vector<int> up, down;
        for (auto &kv : top_of_cap)
            if (ks[kv.second] > k0) up.push_back(kv.second);                // register-cap rungs
        for (int i = 0; i < n; ++i)
            if (ks[i] < k0) down.push_back(i);                              // padding levels
        std::sort(up.begin(), up.end(), [&](int a, int b) { return ks[a] < ks[b]; });
        std::sort(down.begin(), down.end(), [&](int a, int b) { return ks[a] > ks[b]; });
        up.insert(up.begin(), orig);
        down.insert(down.begin(), orig);
        if (natural_regs >= cfg.maxlive_threshold) {       // Fig. 8 lines 01-02, 07-09
            direction = ORION_DIR_INCREASING;
            ladder = up;
            other = down;                                   // fail-safe: pad down
        } else {                                            // lines 03-04, 10-11
            direction = ORION_DIR_DECREASING;
            ladder = down;
            other.assign(up.begin(), up.begin() + std::min<size_t>(2, up.size()));   // original + conservative
        }
        if (cfg.expected_iterations > 0 && cfg.expected_iterations < (int)ladder.size() + 2) {
            final_idx = ladder[0];                          // !canTune: the safe original
            final_iter = 0;
        }
    }

    int select() const
    {
        float b = tried.begin()->second;
        for (auto &kv : tried) b = std::min(b, kv.second);
        int pick = -1;
        for (auto &kv : tried) {
            const int i = kv.first;
            const float t = kv.second;
            if (cfg.select_mode == ORION_SELECT_FASTEST) {
                if (pick < 0 || t < tried.at(pick) || (t == tried.at(pick) && ks[i] < ks[pick])) pick = i;
            } else if (t <= b * (1.0f + cfg.slowdown_tol)) {
                if (pick < 0 || ks[i] < ks[pick] || (ks[i] == ks[pick] && t < tried.at(pick))) pick = i;
            }
        }
        return pick;
    }

    // "Set final kernel" -- or, with the P:L689 augmentation, switch direction once when
    // the original would be final.  Returns true if the final kernel is now set.
    bool set_final()
    {
        const int f = select();
        if (cfg.allow_direction_switch && !switched && f == ladder[0] && other.size() > 1) {
            switched = true;
            direction = -direction;
            std::swap(ladder, other);
            cur = 0;
            return false;
        }
        final_idx = f;
        final_iter = iter;
        return true;
    }

    // Which level runs this iteration, and whether its time must be measured.
    int choose(bool *measure)
    {
        *measure = false;
        if (final_idx >= 0) return final_idx;                      // "Final kernel has been set?"
        if (cur < 0) {                                             // "First iteration?"
            *measure = true;
            return ladder[0];
        }
        if (cur == (int)ladder.size() - 1 && set_final()) return final_idx;   // tried every occ
        *measure = true;
        return ladder[cur + 1];                                    // "Run next kernel"
    }

    // Feed back the measured time of the level chosen with measure = true.
    void observe(int lvl, float ms)
    {
        if (cur < 0) {
            tried[lvl] = ms;
            best = ms;
            cur = 0;
            return;
        }
        const float prev = tried.at(ladder[cur]);
        ++cur;
        tried[lvl] = ms;
        const bool stop = (direction == ORION_DIR_INCREASING) ? ms > prev * (1.0f + cfg.worse_eps)      // "Worse runtime?"
                                                              : ms > best * (1.0f + cfg.slowdown_tol);  // "Slowdown > .02?"
        best = std::min(best, ms);
        if (stop) set_final();
    }
};

orion_status check_cfg(const orion_tuner_cfg *c)
{
    if (!c || c->samples_per_level < 1 || c->slowdown_tol < 0.0f || c->worse_eps < 0.0f ||
        (c->async_timing != 0 && c->async_timing != 1) ||
        (c->select_mode != ORION_SELECT_FASTEST && c->select_mode != ORION_SELECT_LOWEST_WITHIN_TOL))
        return fail(ORION_E_INVALID, "bad tuner cfg");
    return ORION_OK;
}

orion_status check_levels(const orion_level *lv, int n)
{
    if (!lv || n <= 0) return fail(ORION_E_INVALID, "no levels");
    for (int i = 0; i < n; ++i)
        if (lv[i].reg_cap == 0) return ORION_OK;
    return fail(ORION_E_INVALID, "levels lack the original (uncapped) version");
}

}  // namespace

struct orion_tuner {
    orion_variants *v = nullptr;
    Fig9 f;
    CUevent e0 = nullptr, e1 = nullptr;
    int pending_level = -1;      // level being sampled (samples_per_level > 1)
    int samples = 0;
    float sample_best = 0.0f;
    // async_timing: the one measured launch whose event pair has not been read yet
    bool inflight = false;
    int inflight_level = -1;
    double inflight_work = 0.0;
};

extern "C" {

orion_status orion_tuner_default_cfg(orion_tuner_cfg *c)
{
    if (!c) return fail(ORION_E_INVALID, "NULL cfg");
    c->maxlive_threshold = 32;
    c->samples_per_level = 1;
    c->select_mode = ORION_SELECT_FASTEST;
    c->allow_direction_switch = 1;   // P:L689 augmentation on by default (reading R-A12)
    c->slowdown_tol = 0.02f;
    c->worse_eps = 0.0f;
    c->expected_iterations = 0;
    c->async_timing = 0;
    return ORION_OK;
}

orion_status orion_tuner_replay(const orion_tuner_cfg *cfg, const orion_level *levels, int n, int natural_regs,
                                const float *ms_of_level, int iterations, int *ran, int *final_level_idx,
                                int *final_iteration)
{
    ORION_TRY(check_cfg(cfg));
    ORION_TRY(check_levels(levels, n));
    if (!ms_of_level || iterations < 0 || (iterations > 0 && !ran)) return fail(ORION_E_INVALID, "replay: bad argument");
    Fig9 f;
    f.cfg = *cfg;
    f.prune(levels, n, natural_regs);
    for (int it = 0; it < iterations; ++it) {
        f.iter = it;
        bool measure;
        const int lvl = f.choose(&measure);
        if (measure) f.observe(lvl, ms_of_level[lvl]);
        ran[it] = lvl;
    }
    if (final_level_idx) *final_level_idx = f.final_idx;
    if (final_iteration) *final_iteration = f.final_iter;
    return ORION_OK;
}

orion_status orion_tuner_create(orion_variants *v, const orion_tuner_cfg *cfg, orion_tuner **out)
{
    if (!v || !out) return fail(ORION_E_INVALID, "orion_tuner_create: NULL");
    ORION_TRY(check_cfg(cfg));
    std::vector<orion_level> lv(v->vars.size());
    for (size_t i = 0; i < lv.size(); ++i) lv[i] = v->vars[i].planned;
    ORION_TRY(check_levels(lv.data(), (int)lv.size()));
    ORION_TRY(ensure_context(v->device));
    auto t = new orion_tuner();
    t->v = v;
    t->f.cfg = *cfg;
    t->f.prune(lv.data(), (int)lv.size(), v->res.regs_per_thread);
    const Driver &D = drv();
    if (D.cuEventCreate(&t->e0, CU_EVENT_DEFAULT) != CUDA_SUCCESS ||
        D.cuEventCreate(&t->e1, CU_EVENT_DEFAULT) != CUDA_SUCCESS) {
        orion_tuner_destroy(t);
        return fail(ORION_E_CUDA, "cuEventCreate");
    }
    *out = t;
    return ORION_OK;
}

void orion_tuner_destroy(orion_tuner *t)
{
    if (!t) return;
    if (drv().ok) {
        if (t->e0) drv().cuEventDestroy(t->e0);
        if (t->e1) drv().cuEventDestroy(t->e1);
    }
    delete t;
}

// Feed one completed measurement (ms of a launch over `work` output elements) to Fig. 9,
// through the samples_per_level filter (the fastest of the samples is observed).
static void feed_sample(orion_tuner *t, int lvl, float ms, double work)
{
    Fig9 &f = t->f;
    // work-normalised runtime: ns per output element, so iterations of
    // different sizes -- the bands of a split frame -- compare fairly
    const float per = (float)(ms * 1e6 / work);      // work > 0: empty bands never reach here
    const float m = (t->samples == 0) ? per : std::min(t->sample_best, per);
    t->samples += 1;
    t->sample_best = m;
    if (t->samples >= f.cfg.samples_per_level) {
        f.observe(lvl, m);            // best of the samples feeds Fig. 9
        t->pending_level = -1;
        t->samples = 0;
    } else {
        t->pending_level = lvl;
    }
}

orion_status orion_tune_step(orion_tuner *t, const orion_args *a, void *stream, orion_step_report *out)
{
    if (!t || !a) return fail(ORION_E_INVALID, "orion_tune_step: NULL");
    Fig9 &f = t->f;
    CUstream s = (CUstream)stream;
    const Driver &D = drv();
    // output elements of the iteration (every frame of a batch, orion_args.batch)
    const double work = (double)(a->row_end - a->row_begin) * (double)a->width * (double)(a->batch > 1 ? a->batch : 1);
    if (a->row_begin == a->row_end && a->width > 0 && a->row_begin >= 0 && a->row_end <= a->height) {
        // an empty band is not an iteration: nothing is launched, timed or fed to Fig. 9 (a
        // zero-work sample would be in other units than ns per output element)
        if (out) {
            out->iteration = -1;
            out->level_idx = -1;
            out->phase = -1;
            out->final_level_idx = f.final_idx;
            out->ms = -1.0f;
        }
        return ORION_OK;
    }
    float ms = -1.0f;
    auto report = [&](int lvl, int phase) {
        if (out) {
            out->iteration = f.iter;
            out->level_idx = lvl;
            out->phase = phase;
            out->final_level_idx = f.final_idx;
            out->ms = ms;
        }
        f.iter += 1;
        return ORION_OK;
    };
    if (t->inflight) {                    // async_timing: is the measured launch done?
        const CUresult q = D.cuEventQuery(t->e1);
        if (q == CUDA_SUCCESS) {
            ORION_CU(D.cuEventElapsedTime(&ms, t->e0, t->e1));
            t->inflight = false;
            feed_sample(t, t->inflight_level, ms, t->inflight_work);
        } else if (q == CUDA_ERROR_NOT_READY) {
            // not yet: run the level being measured again, untimed (never block the host)
            ORION_TRY(orion_launch(t->v, t->inflight_level, a, stream));
            return report(t->inflight_level, 0);
        } else {
            ORION_CU(q);
        }
    }
    bool measure = false;
    int lvl;
    if (t->pending_level >= 0) {          // still sampling a level (samples_per_level > 1)
        lvl = t->pending_level;
        measure = true;
    } else {
        lvl = f.choose(&measure);
    }
    if (measure) {
        ORION_CU(D.cuEventRecord(t->e0, s));
        ORION_TRY(orion_launch(t->v, lvl, a, stream));
        ORION_CU(D.cuEventRecord(t->e1, s));
        if (f.cfg.async_timing) {
            t->inflight = true;
            t->inflight_level = lvl;
            t->inflight_work = work;
        } else {
            ORION_CU(D.cuEventSynchronize(t->e1));
            ORION_CU(D.cuEventElapsedTime(&ms, t->e0, t->e1));
            feed_sample(t, lvl, ms, work);
        }
    } else {
        ORION_TRY(orion_launch(t->v, lvl, a, stream));
    }
    return report(lvl, measure ? 0 : 1);
}

orion_status orion_tune_steps(orion_tuner *t, const orion_args *args, int n, void *stream, orion_step_report *last)
{
    if (!t || !args || n < 0) return fail(ORION_E_INVALID, "orion_tune_steps: bad argument");
    orion_step_report r{};
    r.level_idx = -1;
    r.ms = -1.0f;
    for (int i = 0; i < n; ++i) ORION_TRY(orion_tune_step(t, &args[i], stream, &r));
    if (last) *last = r;
    return ORION_OK;
}

orion_status orion_tune_split(orion_tuner *t, const orion_args *a, int bands, void *stream, orion_step_report *reports)
{
    if (!t || !a || bands < 1) return fail(ORION_E_INVALID, "orion_tune_split: bad argument");
    const int rows = a->row_end - a->row_begin;
    if (rows < 0) return fail(ORION_E_INVALID, "orion_tune_split: row_end < row_begin");
    const int per = rows > 0 ? (rows + bands - 1) / bands : 0;
    for (int b = 0; b < bands; ++b) {
        orion_args ba = *a;
        ba.row_begin = std::min(a->row_end, a->row_begin + b * per);
        ba.row_end = std::min(a->row_end, ba.row_begin + per);
        orion_step_report r{};
        if (ba.row_begin < ba.row_end) {
            ORION_TRY(orion_tune_step(t, &ba, stream, &r));
        } else {
            r.iteration = -1;
            r.level_idx = -1;
            r.phase = -1;
            r.final_level_idx = t->f.final_idx;
            r.ms = -1.0f;
        }
        if (reports) reports[b] = r;
    }
    return ORION_OK;
}

orion_status orion_tune_step_host(orion_tuner *t, const orion_args *a, void *dev_src, void *dev_dst, void *dev_aux,
                                  void *stream, orion_step_report *out, long long *h2d, long long *d2h)
{
    if (!t || !a || !dev_src || !dev_dst) return fail(ORION_E_INVALID, "orion_tune_step_host: NULL");
    const KernelDef &def = *t->v->def;
    if (def.kind == K_SRAD) return fail(ORION_E_INVALID, "orion_tune_step_host: not available for srad");
    const size_t elem = def.kind == K_STENCIL ? 4 : 16;
    const size_t row = (size_t)a->width * elem;
    // a batch (orion_args.batch, whole frames) is copied as one block of B frames each way
    const size_t nb = a->batch > 1 ? (size_t)a->batch : 1;
    const size_t in_bytes = (size_t)(a->src_row_end - a->src_row_begin) * row * nb;
    const size_t out_bytes = (size_t)(a->row_end - a->row_begin) * row * nb;
    if (a->src_row_end < a->src_row_begin || (def.kind == K_STENCIL && (!dev_aux || !a->aux)))
        return fail(ORION_E_INVALID, "orion_tune_step_host: bad argument");
    const Driver &D = drv();
    CUstream s = (CUstream)stream;
    ORION_TRY(ensure_context(t->v->device));
    ORION_CU(D.cuMemcpyHtoDAsync((CUdeviceptr)dev_src, a->src, in_bytes, s));
    size_t aux_bytes = 0;
    if (def.kind == K_STENCIL) {
        aux_bytes = in_bytes;
        ORION_CU(D.cuMemcpyHtoDAsync((CUdeviceptr)dev_aux, a->aux, aux_bytes, s));
    }
    orion_args da = *a;
    da.src = dev_src;
    da.dst = dev_dst;
    da.aux = dev_aux;
    da.flags = 0;                  // the launch follows this call's own copies
    da.chain = nullptr;
    ORION_TRY(orion_tune_step(t, &da, stream, out));
    const char *dptr = (const char *)dev_dst + (size_t)(a->row_begin - a->dst_row_begin) * row;
    ORION_CU(D.cuMemcpyDtoHAsync((char *)a->dst + (size_t)(a->row_begin - a->dst_row_begin) * row,
                                 (CUdeviceptr)dptr, out_bytes, s));
    ORION_CU(D.cuStreamSynchronize(s));
    if (h2d) *h2d = (long long)(in_bytes + aux_bytes);
    if (d2h) *d2h = (long long)out_bytes;
    return ORION_OK;
}

orion_status orion_tune_run_host(orion_tuner *t, const orion_args *a, int iterations, void *dev_a, void *dev_b,
                                 void *dev_aux, const int *roi, void *stream, long long *h2d, long long *d2h)
{
    if (!t || !a || !dev_a || !dev_b || iterations < 1 || !a->src || !a->dst)
        return fail(ORION_E_INVALID, "orion_tune_run_host: bad argument");
    const KernelDef &def = *t->v->def;
    const bool srad = def.kind == K_SRAD;
    if (def.kind != K_STENCIL && !srad) return fail(ORION_E_INVALID, "orion_tune_run_host: stencil kernels only");
    if (a->row_begin != 0 || a->row_end != a->height || a->src_row_begin != 0 || a->src_row_end != a->height ||
        a->dst_row_begin != 0 || a->width < 1 || a->height < 1)
        return fail(ORION_E_INVALID, "orion_tune_run_host: whole grids only (rows [0, height))");
    const bool fused = srad && def.srad_stats;   // statistics slots travel behind the grids
    if ((!dev_aux && !fused) || (!srad && !a->aux) || (srad && !roi))
        return fail(ORION_E_INVALID, "orion_tune_run_host: missing aux / roi");
    const size_t bytes = (size_t)a->width * (size_t)a->height * 4;
    const Driver &D = drv();
    CUstream s = (CUstream)stream;
    ORION_TRY(ensure_context(t->v->device));
    ORION_CU(D.cuMemcpyHtoDAsync((CUdeviceptr)dev_a, a->src, bytes, s));
    size_t in_bytes = bytes;
    if (!srad) {
        ORION_CU(D.cuMemcpyHtoDAsync((CUdeviceptr)dev_aux, a->aux, bytes, s));
        in_bytes += bytes;
    }
    void *cur = dev_a, *nxt = dev_b;
    if (fused)
        ORION_TRY(orion_srad_stats_init(t->v->device, cur, a->width, a->height, roi[0], roi[1], roi[2], roi[3],
                                        stream));
    // chainable families: the iterations overlap tile by tile (orion_chain); the chain is freed
    // only after the stream has drained, on every path
    struct ChainGuard {
        orion_chain *c = nullptr;
        CUstream s = nullptr;
        ~ChainGuard()
        {
            if (c) {
                drv().cuStreamSynchronize(s);
                orion_chain_destroy(c);
            }
        }
    } chain;
    chain.s = s;
    if (def.chain && a->n_fanout == 0 && a->flags == 0)
        ORION_TRY(orion_chain_create(t->v, a->width, a->height, &chain.c));
    for (int it = 0; it < iterations; ++it) {
        if (srad && !fused)
            ORION_TRY(orion_srad_roi_stats(t->v->device, cur, a->width, a->height, roi[0], roi[1], roi[2], roi[3],
                                           dev_aux, stream));
        orion_args da = *a;
        da.src = cur;
        da.dst = nxt;
        da.aux = dev_aux;
        da.chain = chain.c;
        if (fused)
            for (int i = 0; i < 4; ++i) da.fparam[1 + i] = (float)roi[i];
        ORION_TRY(orion_tune_step(t, &da, stream, nullptr));
        std::swap(cur, nxt);
    }
    ORION_CU(D.cuMemcpyDtoHAsync(a->dst, (CUdeviceptr)cur, bytes, s));
    ORION_CU(D.cuStreamSynchronize(s));
    if (h2d) *h2d = (long long)in_bytes;
    if (d2h) *d2h = (long long)bytes;
    return ORION_OK;
}

}  // extern "C"

// ---- pipelined host-buffer iterations --------------------------------------------------------
// depth slots of library-owned device staging buffers and three library-owned streams:
// H2D of frame n+1 and D2H of frame n-1 overlap the kernel of frame n (PCIe is full duplex).
struct orion_host_pipe {
    orion_tuner *t = nullptr;
    int width = 0, max_rows = 0;
    size_t elem = 16;
    CUstream s_in = nullptr, s_comp = nullptr, s_out = nullptr;
    struct Slot {
        CUdeviceptr src = 0, dst = 0, aux = 0;
        CUevent ev_in = nullptr, ev_done = nullptr, ev_out = nullptr;
        bool used = false;
    };
    std::vector<Slot> slots;
    int next = 0;
};

extern "C" {

void orion_host_pipe_destroy(orion_host_pipe *p)
{
    if (!p) return;
    if (drv().ok) {
        const Driver &D = drv();
        for (CUstream s : {p->s_in, p->s_comp, p->s_out})
            if (s) D.cuStreamSynchronize(s);
        for (auto &s : p->slots) {
            for (CUdeviceptr m : {s.src, s.dst, s.aux})
                if (m) D.cuMemFree(m);
            for (CUevent e : {s.ev_in, s.ev_done, s.ev_out})
                if (e) D.cuEventDestroy(e);
        }
        for (CUstream s : {p->s_in, p->s_comp, p->s_out})
            if (s) D.cuStreamDestroy(s);
    }
    delete p;
}

orion_status orion_host_pipe_create(orion_tuner *t, int width, int max_rows, int depth, orion_host_pipe **out)
{
    if (!t || !out || width <= 0 || max_rows <= 0 || depth < 1 || depth > 8)
        return fail(ORION_E_INVALID, "orion_host_pipe_create: bad argument");
    ORION_TRY(ensure_context(t->v->device));
    const Driver &D = drv();
    auto p = new orion_host_pipe();
    std::unique_ptr<orion_host_pipe, void (*)(orion_host_pipe *)> guard(p, orion_host_pipe_destroy);
    p->t = t;
    p->width = width;
    p->max_rows = max_rows;
    if (t->v->def->kind == K_SRAD) return fail(ORION_E_INVALID, "orion_host_pipe_create: not available for srad");
    const bool stencil = t->v->def->kind == K_STENCIL;
    p->elem = stencil ? 4 : 16;
    const size_t bytes = (size_t)width * (size_t)max_rows * p->elem;
    ORION_CU(D.cuStreamCreate(&p->s_in, CU_STREAM_NON_BLOCKING));
    ORION_CU(D.cuStreamCreate(&p->s_comp, CU_STREAM_NON_BLOCKING));
    ORION_CU(D.cuStreamCreate(&p->s_out, CU_STREAM_NON_BLOCKING));
    p->slots.resize(depth);
    for (auto &s : p->slots) {
        ORION_CU(D.cuMemAlloc(&s.src, bytes));
        ORION_CU(D.cuMemAlloc(&s.dst, bytes));
        if (stencil) ORION_CU(D.cuMemAlloc(&s.aux, bytes));
        ORION_CU(D.cuEventCreate(&s.ev_in, CU_EVENT_DISABLE_TIMING));
        ORION_CU(D.cuEventCreate(&s.ev_done, CU_EVENT_DISABLE_TIMING));
        ORION_CU(D.cuEventCreate(&s.ev_out, CU_EVENT_DISABLE_TIMING));
    }
    *out = guard.release();
    return ORION_OK;
}

orion_status orion_host_pipe_submit(orion_host_pipe *p, const orion_args *a, orion_step_report *out,
                                    long long *h2d, long long *d2h)
{
    if (!p || !a || !a->src || !a->dst) return fail(ORION_E_INVALID, "orion_host_pipe_submit: NULL");
    // a batch (orion_args.batch, whole frames) occupies B frames' rows of a slot
    const int nb = a->batch > 1 ? a->batch : 1;
    const long long in_rows_ll = (long long)(a->src_row_end - a->src_row_begin) * nb;
    const long long out_rows_ll = (long long)(a->row_end - a->row_begin) * nb;
    if (in_rows_ll > p->max_rows || out_rows_ll > p->max_rows)
        return fail(ORION_E_INVALID, "orion_host_pipe_submit: frame does not fit the pipe");
    const int in_rows = (int)in_rows_ll;
    const int out_rows = (int)out_rows_ll;
    if (a->width != p->width || in_rows < 0 || in_rows > p->max_rows || out_rows < 0 || out_rows > p->max_rows ||
        a->dst_row_begin > a->row_begin || (p->t->v->def->kind == K_STENCIL && !a->aux))
        return fail(ORION_E_INVALID, "orion_host_pipe_submit: frame does not fit the pipe");
    const Driver &D = drv();
    ORION_TRY(ensure_context(p->t->v->device));
    auto &s = p->slots[p->next];
    p->next = (p->next + 1) % (int)p->slots.size();
    const size_t row = (size_t)a->width * p->elem;
    const size_t in_bytes = (size_t)in_rows * row, out_bytes = (size_t)out_rows * row;
    if (s.used) ORION_CU(D.cuStreamWaitEvent(p->s_in, s.ev_out, 0));   // slot free again
    ORION_CU(D.cuMemcpyHtoDAsync(s.src, a->src, in_bytes, p->s_in));
    size_t aux_bytes = 0;
    if (s.aux) {
        aux_bytes = in_bytes;
        ORION_CU(D.cuMemcpyHtoDAsync(s.aux, a->aux, aux_bytes, p->s_in));
    }
    ORION_CU(D.cuEventRecord(s.ev_in, p->s_in));
    ORION_CU(D.cuStreamWaitEvent(p->s_comp, s.ev_in, 0));
    orion_args da = *a;
    da.src = (const void *)s.src;
    da.dst = (void *)s.dst;
    da.aux = (const void *)s.aux;
    da.flags = 0;                  // the launch follows the pipe's copies and event waits
    da.chain = nullptr;
    da.dst_row_begin = a->row_begin;
    ORION_TRY(orion_tune_step(p->t, &da, p->s_comp, out));
    ORION_CU(D.cuEventRecord(s.ev_done, p->s_comp));
    ORION_CU(D.cuStreamWaitEvent(p->s_out, s.ev_done, 0));
    ORION_CU(D.cuMemcpyDtoHAsync((char *)a->dst + (size_t)(a->row_begin - a->dst_row_begin) * row, s.dst, out_bytes,
                                 p->s_out));
    ORION_CU(D.cuEventRecord(s.ev_out, p->s_out));
    s.used = true;
    if (h2d) *h2d = (long long)(in_bytes + aux_bytes);
    if (d2h) *d2h = (long long)out_bytes;
    return ORION_OK;
}

orion_status orion_host_pipe_drain(orion_host_pipe *p)
{
    if (!p) return fail(ORION_E_INVALID, "orion_host_pipe_drain: NULL");
    ORION_TRY(ensure_context(p->t->v->device));
    const Driver &D = drv();
    ORION_CU(D.cuStreamSynchronize(p->s_in));
    ORION_CU(D.cuStreamSynchronize(p->s_comp));
    ORION_CU(D.cuStreamSynchronize(p->s_out));
    return ORION_OK;
}

orion_status orion_tuner_ladder(const orion_tuner *t, int *direction, int *out, int capacity, int *n_out)
{
    if (!t || !n_out || capacity < 0 || (capacity > 0 && !out)) return fail(ORION_E_INVALID, "orion_tuner_ladder");
    if (direction) *direction = t->f.direction;
    *n_out = (int)t->f.ladder.size();
    if ((int)t->f.ladder.size() > capacity) return fail(ORION_E_CAPACITY, "orion_tuner_ladder: capacity");
    std::copy(t->f.ladder.begin(), t->f.ladder.end(), out);
    return ORION_OK;
}

orion_status orion_tuner_resume(orion_tuner *t, int final_level_idx)
{
    if (!t) return fail(ORION_E_INVALID, "orion_tuner_resume: NULL");
    if (final_level_idx < 0 || final_level_idx >= (int)t->v->vars.size())
        return fail(ORION_E_INVALID, "orion_tuner_resume: level index out of range");
    if (t->inflight) return fail(ORION_E_STATE, "orion_tuner_resume: a measurement is in flight");
    t->f.final_idx = final_level_idx;
    t->f.final_iter = t->f.iter;
    t->pending_level = -1;
    t->samples = 0;
    return ORION_OK;
}

orion_status orion_tuner_tried(const orion_tuner *t, float *out, int n)
{
    if (!t || !out || n != (int)t->v->vars.size()) return fail(ORION_E_INVALID, "orion_tuner_tried: bad argument");
    for (int i = 0; i < n; ++i) out[i] = -1.0f;
    for (auto &kv : t->f.tried) out[kv.first] = kv.second;
    return ORION_OK;
}

orion_status orion_tuner_final(const orion_tuner *t, int *final_level_idx, int *iterations_to_final)
{
    if (!t) return fail(ORION_E_INVALID, "orion_tuner_final: NULL");
    if (final_level_idx) *final_level_idx = t->f.final_idx;
    if (iterations_to_final) *iterations_to_final = t->f.final_iter;
    return ORION_OK;
}

}  // extern "C"

struct orion_graph {
    orion_tuner *t = nullptr;
    CUgraph graph = nullptr;
    CUgraphExec exec = nullptr;
    int n = 0;
};

extern "C" {

void orion_graph_destroy(orion_graph *g)
{
    if (!g) return;
    if (drv().ok) {
        if (g->exec) drv().cuGraphExecDestroy(g->exec);
        if (g->graph) drv().cuGraphDestroy(g->graph);
    }
    delete g;
}

orion_status orion_tuner_capture(orion_tuner *t, const orion_args *args, int n, orion_graph **out)
{
    if (!t || !args || n < 1 || !out) return fail(ORION_E_INVALID, "orion_tuner_capture: bad argument");
    *out = nullptr;
    if (t->f.final_idx < 0 || t->inflight) return fail(ORION_E_STATE, "orion_tuner_capture: the tuner is still exploring");
    ORION_TRY(ensure_context(t->v->device));
    const Driver &D = drv();
    CUstream s = nullptr;
    ORION_CU(D.cuStreamCreate(&s, CU_STREAM_NON_BLOCKING));
    std::unique_ptr<orion_graph, void (*)(orion_graph *)> g(new orion_graph(), orion_graph_destroy);
    g->t = t;
    g->n = n;
    orion_status st = ORION_OK;
    if (D.cuStreamBeginCapture(s, CU_STREAM_CAPTURE_MODE_THREAD_LOCAL) != CUDA_SUCCESS)
        st = fail(ORION_E_CUDA, "cuStreamBeginCapture");
    const long long before = g_launches.load();
    // graph nodes are plain kernel launches, unless every captured launch is independent
    // (ORION_ARGS_INDEPENDENT): then they keep programmatic dependent launch, the graph gets
    // programmatic edges and, as the kernels skip griddepcontrol.wait, consecutive frames run
    // concurrently (C1: 2.9 -> 1.3 us per 64^2 frame; with waiting kernels the edges measured
    // ~4.0 vs ~3.8 us, no gain)
    bool indep = true;
    for (int i = 0; i < n; ++i) indep = indep && (args[i].flags & ORION_ARGS_INDEPENDENT);
    t_capturing = true;
    t_capture_pdl = indep;
    for (int i = 0; i < n && st == ORION_OK; ++i) st = orion_launch(t->v, t->f.final_idx, &args[i], s);
    t_capturing = false;
    t_capture_pdl = false;
    g_launches.store(before);   // captured, not launched: replays are counted
    CUgraph graph = nullptr;
    const CUresult end = D.cuStreamEndCapture(s, &graph);   // always end the capture
    g->graph = graph;
    if (st == ORION_OK && end != CUDA_SUCCESS) st = fail(ORION_E_CUDA, "cuStreamEndCapture");
    if (st == ORION_OK && D.cuGraphInstantiate(&g->exec, g->graph, 0) != CUDA_SUCCESS)
        st = fail(ORION_E_CUDA, "cuGraphInstantiate");
    D.cuStreamDestroy(s);
    if (st != ORION_OK) return st;
    *out = g.release();
    return ORION_OK;
}

orion_status orion_graph_launch(orion_graph *g, void *stream)
{
    if (!g || !g->exec) return fail(ORION_E_INVALID, "orion_graph_launch: NULL");
    ORION_TRY(ensure_context(g->t->v->device));
    ORION_CU(drv().cuGraphLaunch(g->exec, (CUstream)stream));
    g_launches.fetch_add(g->n);
    g->t->f.iter += g->n;
    return ORION_OK;
}

}  // extern "C"
