// model.cu -- the paper's advanced hybrid work-division model.
//
// Sec. 5.2: on an HPU with p CPU cores, g GPU cores and CPU/GPU
// speed ratio gamma (Sec. 3.2), a fraction alpha of the
// subproblems of a D&C T(n) = aT(n/b) + f(n), f(m) = m^{log_b a}, runs on
// the CPU, the rest on the GPU from the leaves up to level y, chosen so both
// finish together; alpha is chosen to maximise the GPU's share of the work.
// Host-only arithmetic in double precision; no device work.  (On a B200 box
// every level runs on the GPUs -- DESIGN.md Sec. 7 -- so this model is the
// paper's analysis made callable, pinned by its printed example.)
#include <cmath>

#include "dc.h"
#include "plan.h"

namespace {

double logb_(double x, double base) { return std::log(x) / std::log(base); }

struct ModelEval {
    double frac, y;
    int kase;
};

// Closed forms of Sec. 5.2.2: Tc, Tmaxg, the three cases of Tg,
// y solving Tg = Tc, and the GPU work Wg = (1-alpha) N (L - y + 1) relative
// to the total N (L + 1).
ModelEval evaluate(double a, double b, double p, double g, double gamma, double n, double alpha) {
    const double N = std::pow(n, logb_(a, b));
    const double L = logb_(n, b);
    const double Tc = alpha * N / p * (L - logb_(p / alpha, a) + 1.0);
    const double Tmaxg = (1.0 - alpha) * N / (gamma * g) * (L - logb_(g / (1.0 - alpha), a) + 1.0);
    ModelEval r{};
    if ((1.0 - alpha) * N < g) {                   // (i) the GPU never saturates
        const double ay = (gamma * Tc + 1.0 / (a - 1.0)) * (a - 1.0) / (N * a);
        r.y = -logb_(ay, a);
        r.kase = 1;
    } else if (Tmaxg >= Tc) {                      // (ii) always saturated
        r.y = L + 1.0 - Tc * gamma * g / ((1.0 - alpha) * N);
        r.kase = 2;
    } else {                                       // (iii) saturated, then not
        const double ay = (Tc - Tmaxg) * gamma * (a - 1.0) / (N * a) + (1.0 - alpha) / g;
        r.y = -logb_(ay, a);
        r.kase = 3;
    }
    r.frac = (1.0 - alpha) * (L - r.y + 1.0) / (L + 1.0);
    return r;
}

bool valid(int32_t a, int32_t b, int32_t p, double g, double gamma, double n) {
    return a >= 2 && b >= 2 && p >= 1 && g >= 1.0 && gamma > 0.0 && gamma < 1.0 && n >= 2.0 &&
           std::isfinite(g) && std::isfinite(n);
}

}  // namespace

extern "C" {

dc_status dc_model_gpu_work(int32_t a, int32_t b, int32_t p, double g, double gamma, double n,
                            double alpha, double* gpu_work_fraction, double* level_y,
                            int32_t* model_case) {
    if (!valid(a, b, p, g, gamma, n)) return DC_ERR_INVALID_ARG;
    const double N = std::pow(n, logb_(a, b));
    if (!(alpha >= p / N && alpha < 1.0)) return DC_ERR_INVALID_ARG;   // alpha >= p/n
    const ModelEval r = evaluate(a, b, p, g, gamma, n, alpha);
    if (gpu_work_fraction) *gpu_work_fraction = r.frac;
    if (level_y) *level_y = r.y;
    if (model_case) *model_case = r.kase;
    return DC_OK;
}

dc_status dc_model_optimise(int32_t a, int32_t b, int32_t p, double g, double gamma, double n,
                            double* alpha, double* gpu_work_fraction, double* level_y,
                            int32_t* model_case) {
    if (!valid(a, b, p, g, gamma, n)) return DC_ERR_INVALID_ARG;
    // "maximize the work using numeric methods": a uniform scan of
    // alpha in [p/N, 1), then golden-section refinement around the best point.
    const double N = std::pow(n, logb_(a, b));
    const double lo = p / N;
    const int steps = 4096;
    double best_a = lo, best_f = -1.0;
    for (int k = 1; k < steps; ++k) {
        const double al = lo + (1.0 - lo) * k / steps;
        const double f = evaluate(a, b, p, g, gamma, n, al).frac;
        if (f > best_f) {
            best_f = f;
            best_a = al;
        }
    }
    double x0 = std::fmax(lo, best_a - (1.0 - lo) / steps);
    double x1 = std::fmin(1.0 - 1e-12, best_a + (1.0 - lo) / steps);
    const double phi = 0.5 * (std::sqrt(5.0) - 1.0);
    for (int it = 0; it < 80; ++it) {
        const double c = x1 - phi * (x1 - x0), d = x0 + phi * (x1 - x0);
        if (evaluate(a, b, p, g, gamma, n, c).frac >= evaluate(a, b, p, g, gamma, n, d).frac) x1 = d;
        else x0 = c;
    }
    const double al = 0.5 * (x0 + x1);
    const ModelEval r = evaluate(a, b, p, g, gamma, n, al);
    const ModelEval rb = evaluate(a, b, p, g, gamma, n, best_a);
    const bool use_scan = rb.frac > r.frac;        // a case boundary can break unimodality
    if (alpha) *alpha = use_scan ? best_a : al;
    if (gpu_work_fraction) *gpu_work_fraction = use_scan ? rb.frac : r.frac;
    if (level_y) *level_y = use_scan ? rb.y : r.y;
    if (model_case) *model_case = use_scan ? rb.kase : r.kase;
    return DC_OK;
}

}  // extern "C"

// ===================================================================
// B200 schedule planner: the Sec. 5.2 analysis re-parameterised.
//
// The paper assigns the levels of the recursion tree of T(n) = aT(n/b) + f(n)
// to processing units with different per-level speeds and parallelism
// thresholds (p CPU cores, g GPU cores, speed ratio gamma; a unit pays off at
// a level only when that level has enough subproblems to saturate it,
// P:L432-433), and chooses the split (alpha, y) from closed-form
// level costs.  On one B200 the "units" are the levels a sort
// can run on:
//   * on chip (NK1): the bottom ceil(log2 T) levels of every tile, T fixed by
//     the compiled tile class (quarter-size: 128-thread CTAs, full: 512 or
//     256 threads) -- a level here costs shared-memory wavefronts, not HBM;
//   * HBM passes above the tile: one level per pass (NK2 + NK3) or two levels
//     per pass (NK2-4 + NK3-4, f1);
// and the parallelism threshold is the SM count: a pass whose launch has
// fewer CTAs than resident slots, or whose data stays in L2, runs in a
// different regime (latency / L2 bandwidth) than a saturated HBM pass.  The
// level table gives, for each candidate (tile class, pass kind), how many
// levels run where (fused = ceil(log2 T), P = ceil(log2(n / T)) global
// levels, P/2 two-level passes + P mod 2 one-level passes); each unit's cost
// is affine in the keys it moves, with a per-launch term, fitted to B200
// measurements of whole sorts (tools/planner_sweep.py ->
// profiles/r02/planner_sweep.json, fit in tools/planner_fit.py).  The plan
// runs the candidate of least predicted time: that is the Sec. 5.2 step
// "maximise with numeric methods" with time as the objective,
// because on one GPU the units run one after another instead of side by side.
namespace {

// Cost of one kernel of the schedule: c0 + W * wave, W = ceil(ctas / slots)
// waves of resident CTAs, each costing `wave` ms (the time a resident CTA
// needs for its tile: the shared-memory- and latency-bound kernels pay per
// wave; for the HBM-bound one-level pass the wave time absorbs bandwidth);
// `wave` has an L2-resident and an HBM-resident value (the level's 8n bytes,
// 16n with values, within kPlannerL2Bytes or not).
struct KCost {
    double c0;                  // ms per launch (latency of the first wave, launch gap)
    double wave_l2, wave_hbm;   // ms per wave
    int slots;                  // resident CTAs per wave (SMs x CTAs per SM)
    int tile;                   // keys per CTA tile (outputs for merges)
};
struct ClassCost {
    KCost nk1[2];               // [quarter tiles, full tiles]
    KCost pass1[2];             // one-level merge pass (NK3; quarter tiles: partition fused)
    double nk2_0, nk2_t;        // separate NK2 of a full-tile one-level pass: c0 + per tile
    KCost merge4;               // two-level pass: persistent 4-way tile merge
    double sel_0, sel_t;        // NK2-4 (exact 4-run cuts): c0 + per 4-way tile
};

#include "planner_coeffs.inc"    // kPlannerCost[3] (keys-only, f32 keys, key-value), kPlannerL2Bytes

double waves(int64_t ctas, int slots) { return (double)((ctas + slots - 1) / slots); }

int global_levels(int64_t n, int64_t tile) {
    int p = 0;
    for (int64_t w = tile; w < n; w *= 2) ++p;
    return p;
}

double predict(int cls, int64_t n, bool small, bool two, int* hbm_passes, int* tile_out) {
    const ClassCost& c = kPlannerCost[cls];
    const int s = small ? 0 : 1;
    const int tile = c.nk1[s].tile;
    const int P = global_levels(n, tile);
    const bool use_two = two && P >= 2;
    const int single = use_two ? P % 2 : P;
    const int doubles = use_two ? (P - single) / 2 : 0;
    const bool l2 = 8.0 * (double)n * (cls == 2 ? 2.0 : 1.0) <= kPlannerL2Bytes;
    auto run = [&](const KCost& k, int64_t ctas) {
        return k.c0 + waves(ctas, k.slots) * (l2 ? k.wave_l2 : k.wave_hbm);
    };
    double t = run(c.nk1[s], (n + tile - 1) / tile);
    const int64_t t1 = (n + c.pass1[s].tile - 1) / c.pass1[s].tile;
    for (int i = 0; i < single; ++i) {
        t += run(c.pass1[s], t1);
        if (!small) t += c.nk2_0 + c.nk2_t * (double)t1;
    }
    const int64_t t4 = (n + c.merge4.tile - 1) / c.merge4.tile;
    for (int i = 0; i < doubles; ++i) t += run(c.merge4, t4) + c.sel_0 + c.sel_t * (double)t4;
    if (hbm_passes) *hbm_passes = single + doubles;
    if (tile_out) *tile_out = tile;
    return t;
}

}  // namespace

extern "C" {

dc_status dc_model_sort_schedule(int64_t n, dc_key_type key_type, int32_t with_vals,
                                 int32_t tile_class, int32_t two_level, dc_sort_schedule* out) {
    if (!out || n < 1 || n > 2147483647LL ||
        (key_type != DC_KEY_U32 && key_type != DC_KEY_I32 && key_type != DC_KEY_F32) ||
        tile_class < 0 || tile_class > 2 || two_level < -1 || two_level > 1)
        return dcx::fail(DC_ERR_INVALID_ARG, "bad schedule-model arguments");
    const int cls = with_vals ? 2 : (key_type == DC_KEY_F32 ? 1 : 0);
    *out = dc_sort_schedule{};
    // every candidate's prediction; the allowed ones compete
    double t[4];
    int hp[4], tl[4];
    bool ok[4];
    double best = 1e300;
    for (int sm = 0; sm < 2; ++sm) {
        for (int tw = 0; tw < 2; ++tw) {
            const int i = 2 * sm + tw;
            t[i] = predict(cls, n, sm == 0, tw == 1, &hp[i], &tl[i]);
            out->candidates_ms[i] = t[i];
            ok[i] = !((tile_class == 1 && sm != 0) || (tile_class == 2 && sm == 0) ||
                      (two_level >= 0 && tw != two_level));
            if (ok[i] && t[i] < best) best = t[i];
        }
    }
    // The least predicted time wins; within the model's resolution (3 %, the
    // fit's median error is 2-4 %) a full-tile schedule with the same number
    // of HBM passes is preferred (it keeps more levels on chip; the measured
    // sweep favours it at every such near-tie: key-value 2^24..2^28).
    int pick = -1;
    for (int i = 0; i < 4; ++i)
        if (ok[i] && (pick < 0 || t[i] < t[pick])) pick = i;
    if (pick / 2 == 0) {
        const int full = 2 + pick % 2;
        if (ok[full] && hp[full] == hp[pick] && t[full] <= t[pick] * 1.03) pick = full;
    }
    out->tile_class = pick / 2 == 0 ? 1 : 2;
    out->two_level = pick % 2;
    out->tile = tl[pick];
    out->global_levels = global_levels(n, tl[pick]);
    out->hbm_passes = hp[pick];
    out->predicted_ms = t[pick];
    int f = 0;
    while ((1 << f) < out->tile) ++f;
    out->fused_levels = f;
    return DC_OK;
}

}  // extern "C"
