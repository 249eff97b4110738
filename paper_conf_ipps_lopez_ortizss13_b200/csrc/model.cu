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
