// schedule.cpp -- viper_schedule: the Inference Performance Predictor
// (PAPER.md s4.3 "Optimized Checkpointing Schedule"), host only.
//
//   TLP    fit Exp2 a e^{-bx}, Exp3 a e^{-bx}+c, Lin2 a x+b, Expd3 c-(c-a)e^{-bx}
//          to the warm-up losses, keep the min-MSE family;
//          ties within rel 1e-9 go to the paper's list order (R7).
//          Exponentials: Levenberg-Marquardt with analytic Jacobians from two
//          starting points (R9); Lin2: closed-form least squares.
//   t_p = s_model / bw_write, t_c = s_model / bw_read
//   Alg. 1 CIL (R1), Alg. 2 fixed interval (R2, R6),
//   Alg. 3 greedy irregular (R3), threshold = mean + std of
//   |consecutive warm-up loss differences| (R8).
#include <cmath>
#include <cstring>
#include <limits>
#include <vector>

#include "../../include/viper.h"
#include "runtime.h"

namespace vp {
namespace {

int nparams(int fam) { return (fam == VIPER_TLP_EXP2 || fam == VIPER_TLP_LIN2) ? 2 : 3; }

double model_eval(int fam, const double *p, double x) {
    switch (fam) {
        case VIPER_TLP_EXP2: return p[0] * std::exp(-p[1] * x);
        case VIPER_TLP_EXP3: return p[0] * std::exp(-p[1] * x) + p[2];
        case VIPER_TLP_LIN2: return p[0] * x + p[1];
        default: return p[2] - (p[2] - p[0]) * std::exp(-p[1] * x);
    }
}

void model_grad(int fam, const double *p, double x, double *g) {
    const double e = std::exp(-p[1] * x);
    switch (fam) {
        case VIPER_TLP_EXP2: g[0] = e; g[1] = -p[0] * x * e; break;
        case VIPER_TLP_EXP3: g[0] = e; g[1] = -p[0] * x * e; g[2] = 1.0; break;
        case VIPER_TLP_LIN2: g[0] = x; g[1] = 1.0; break;
        default: g[0] = e; g[1] = (p[2] - p[0]) * x * e; g[2] = 1.0 - e; break;
    }
}

double sse(int fam, const double *p, const double *x, const double *y, int n) {
    double s = 0;
    for (int i = 0; i < n; i++) {
        const double r = y[i] - model_eval(fam, p, x[i]);
        s += r * r;
    }
    return s;
}

// Solve A d = b (k x k, k <= 3) by Gaussian elimination with partial pivoting.
bool solve(int k, double A[3][3], double *b, double *d) {
    for (int c = 0; c < k; c++) {
        int piv = c;
        for (int r = c + 1; r < k; r++)
            if (std::fabs(A[r][c]) > std::fabs(A[piv][c])) piv = r;
        if (std::fabs(A[piv][c]) < 1e-300) return false;
        if (piv != c) {
            for (int j = 0; j < k; j++) std::swap(A[c][j], A[piv][j]);
            std::swap(b[c], b[piv]);
        }
        for (int r = c + 1; r < k; r++) {
            const double f = A[r][c] / A[c][c];
            for (int j = c; j < k; j++) A[r][j] -= f * A[c][j];
            b[r] -= f * b[c];
        }
    }
    for (int c = k - 1; c >= 0; c--) {
        double s = b[c];
        for (int j = c + 1; j < k; j++) s -= A[c][j] * d[j];
        d[c] = s / A[c][c];
    }
    return true;
}

// Levenberg-Marquardt from p (in/out).  Returns the final SSE.
double levenberg_marquardt(int fam, double *p, const double *x, const double *y, int n) {
    const int k = nparams(fam);
    double lambda = 1e-3;
    double cur = sse(fam, p, x, y, n);
    for (int iter = 0; iter < 5000 && std::isfinite(cur); iter++) {
        double JTJ[3][3] = {{0}}, JTr[3] = {0}, g[3];
        for (int i = 0; i < n; i++) {
            model_grad(fam, p, x[i], g);
            const double r = y[i] - model_eval(fam, p, x[i]);
            for (int a = 0; a < k; a++) {
                JTr[a] += g[a] * r;
                for (int b = 0; b < k; b++) JTJ[a][b] += g[a] * g[b];
            }
        }
        bool improved = false;
        while (lambda < 1e20) {
            double A[3][3], rhs[3], d[3] = {0, 0, 0};
            for (int a = 0; a < k; a++) {
                for (int b = 0; b < k; b++) A[a][b] = JTJ[a][b];
                A[a][a] += lambda * (JTJ[a][a] > 0 ? JTJ[a][a] : 1e-12);
                rhs[a] = JTr[a];
            }
            if (!solve(k, A, rhs, d)) {
                lambda *= 10;
                continue;
            }
            double q[3] = {p[0], p[1], p[2]};
            for (int a = 0; a < k; a++) q[a] += d[a];
            const double s = sse(fam, q, x, y, n);
            if (std::isfinite(s) && s < cur) {
                double step = 0, norm = 0;
                for (int a = 0; a < k; a++) {
                    step += d[a] * d[a];
                    norm += p[a] * p[a];
                }
                const double rel = (cur - s) / (cur > 0 ? cur : 1);
                for (int a = 0; a < k; a++) p[a] = q[a];
                cur = s;
                lambda = std::max(lambda / 10, 1e-15);
                improved = true;
                if (rel < 1e-15 || step < 1e-30 * (norm + 1e-30)) return cur;
                break;
            }
            lambda *= 10;
        }
        if (!improved) break;
    }
    return cur;
}

void fit_family(int fam, const double *x, const double *y, int n, double *params, double *mse) {
    params[0] = params[1] = params[2] = 0;
    if (fam == VIPER_TLP_LIN2) {  // closed-form least squares
        double sx = 0, sy = 0, sxx = 0, sxy = 0;
        for (int i = 0; i < n; i++) {
            sx += x[i];
            sy += y[i];
            sxx += x[i] * x[i];
            sxy += x[i] * y[i];
        }
        const double mx = sx / n, my = sy / n;
        double vxx = 0, vxy = 0;
        for (int i = 0; i < n; i++) {
            vxx += (x[i] - mx) * (x[i] - mx);
            vxy += (x[i] - mx) * (y[i] - my);
        }
        params[0] = vxx > 0 ? vxy / vxx : 0.0;
        params[1] = my - params[0] * mx;
        *mse = sse(fam, params, x, y, n) / n;
        return;
    }
    // starting points (R9): ones, and one derived from the data
    const double y0 = y[0], y1 = y[n - 1];
    const double span = n > 1 ? x[n - 1] - x[0] : 1.0;
    const double b0 = 1.0 / std::max(span, 1.0);
    double starts[2][3] = {{1, 1, 1}, {0, 0, 0}};
    if (fam == VIPER_TLP_EXP2) { starts[1][0] = std::max(y0, 1e-12); starts[1][1] = b0; }
    else if (fam == VIPER_TLP_EXP3) { starts[1][0] = y0 - y1; starts[1][1] = b0; starts[1][2] = y1; }
    else { starts[1][0] = y0; starts[1][1] = b0; starts[1][2] = y1; }
    double best = std::numeric_limits<double>::infinity();
    for (auto &s0 : starts) {
        double p[3] = {s0[0], s0[1], s0[2]};
        if (nparams(fam) == 2) p[2] = 0;
        const double s = levenberg_marquardt(fam, p, x, y, n);
        if (std::isfinite(s) && s < best) {
            best = s;
            std::memcpy(params, p, sizeof p);
        }
    }
    *mse = std::isfinite(best) ? best / n : std::numeric_limits<double>::infinity();
}

bool mse_equal(double a, double b) {
    return std::fabs(a - b) <= std::max(1e-15, 1e-9 * std::max(std::fabs(a), std::fabs(b)));
}

struct Costs {
    double t_train, t_p, t_c, t_infer;
};

// Algorithm 1; line 8 read as acc_infer_loss <- loss * infers (R1).
void cil(int64_t inter, double loss, int64_t ckpt_ver, int64_t rem, const Costs &c, double *acc, int64_t *infers) {
    double v = ckpt_ver == 1 ? (inter * c.t_train + c.t_p + c.t_c) / c.t_infer : (inter * c.t_train + c.t_p) / c.t_infer;
    int64_t inf = (int64_t)std::floor(v);
    if (inf > rem) inf = rem;
    *acc = loss * (double)inf;
    *infers = inf;
}

}  // namespace
}  // namespace vp

using namespace vp;

extern "C" viper_status viper_schedule(const viper_sched_in *in, viper_sched_out *out) {
    if (!in || !out) return set_error(VIPER_E_INVAL, "null argument");
    if (in->family < 0 && (!in->losses || in->n < 3)) return set_error(VIPER_E_INVAL, "need >= 3 warm-up losses");
    if (in->family > 3) return set_error(VIPER_E_INVAL, "bad family");
    if (in->e_iter < in->s_iter) return set_error(VIPER_E_INVAL, "e_iter < s_iter");
    if (!(in->t_train > 0) || !(in->t_infer > 0)) return set_error(VIPER_E_INVAL, "t_train and t_infer must be > 0");
    if (in->algo != VIPER_SCHED_FIXED && in->algo != VIPER_SCHED_GREEDY) return set_error(VIPER_E_INVAL, "bad algo");
    if (in->total_infers < 0) return set_error(VIPER_E_INVAL, "total_infers < 0");
    Costs c{in->t_train, in->t_p, in->t_c, in->t_infer};
    if (c.t_p < 0) {
        if (!(in->bw_write > 0)) return set_error(VIPER_E_INVAL, "need t_p or bw_write");
        c.t_p = in->s_model / in->bw_write;
    }
    if (c.t_c < 0) {
        if (!(in->bw_read > 0)) return set_error(VIPER_E_INVAL, "need t_c or bw_read");
        c.t_c = in->s_model / in->bw_read;
    }
    // ---- TLP
    std::vector<double> xs;
    if (in->losses && in->n > 0) {
        xs.resize(in->n);
        for (int i = 0; i < in->n; i++) xs[i] = in->x ? in->x[i] : (double)i;
    }
    int fam = in->family;
    double params[3] = {0, 0, 0};
    for (int f = 0; f < 4; f++) out->mse[f] = std::numeric_limits<double>::quiet_NaN();
    if (fam < 0) {
        double p[4][3];
        for (int f = 0; f < 4; f++) fit_family(f, xs.data(), in->losses, in->n, p[f], &out->mse[f]);
        fam = 0;
        for (int f = 1; f < 4; f++)
            if (out->mse[f] < out->mse[fam] && !mse_equal(out->mse[f], out->mse[fam])) fam = f;
        std::memcpy(params, p[fam], sizeof params);
    } else {
        std::memcpy(params, in->params, sizeof params);
    }
    if (!std::isfinite(params[0]) || !std::isfinite(params[1]) || !std::isfinite(params[2]))
        return set_error(VIPER_E_INVAL, "TLP fit failed");
    out->family = fam;
    std::memcpy(out->params, params, sizeof params);
    out->t_p = c.t_p;
    out->t_c = c.t_c;
    auto L = [&](int64_t it) { return model_eval(fam, params, (double)it); };

    std::vector<int64_t> sched;
    const int64_t s = in->s_iter, e = in->e_iter, total = in->total_infers;
    if (in->algo == VIPER_SCHED_FIXED) {  // Algorithm 2
        double min_loss = std::numeric_limits<double>::infinity();
        int64_t best = 0;
        const int64_t max_inter = e - s;
        for (int64_t i = 1; i <= max_inter; i++) {
            double t_l = 0;
            int64_t rem = total;
            double p_l = L(s);
            int64_t c_iter = s + i, ver = 1;
            while (c_iter <= e) {
                double il;
                int64_t inf;
                cil(i, p_l, ver, rem, c, &il, &inf);
                t_l += il;
                rem -= inf;
                p_l = L(c_iter);
                c_iter += i;
                ver++;
            }
            t_l += p_l * (double)rem;
            if (t_l < min_loss) {
                min_loss = t_l;
                best = i;
            }
        }
        out->best_interval = best;
        out->predicted_cil = max_inter >= 1 ? min_loss : L(s) * (double)total;
        out->thresh = 0;
        if (best > 0)
            for (int64_t it = s + best; it <= e; it += best) sched.push_back(it);
    } else {  // Algorithm 3 (R3: i advances every iteration)
        double thresh = in->thresh;
        if (thresh < 0) {
            if (!in->losses || in->n < 2) return set_error(VIPER_E_INVAL, "greedy threshold needs warm-up losses");
            double mean = 0;
            const int nd = in->n - 1;
            std::vector<double> d(nd);
            for (int j = 0; j < nd; j++) {
                d[j] = std::fabs(in->losses[j + 1] - in->losses[j]);
                mean += d[j];
            }
            mean /= nd;
            double var = 0;
            for (int j = 0; j < nd; j++) var += (d[j] - mean) * (d[j] - mean);
            thresh = mean + std::sqrt(var / nd);
        }
        out->thresh = thresh;
        int64_t p_iter = s, i = s + 1, ckpt_v = 1, rem = total;
        double p_l = L(s), acc = 0;
        while (i <= e) {
            const double c_l = L(i);
            if (c_l < p_l && std::fabs(c_l - p_l) > thresh) {
                double il;
                int64_t inf;
                cil(i - p_iter, p_l, ckpt_v, rem, c, &il, &inf);
                acc += il;
                p_l = c_l;
                p_iter = i;
                sched.push_back(i);
                ckpt_v++;
                rem -= inf;
            }
            i++;
        }
        out->best_interval = 0;
        out->predicted_cil = acc + p_l * (double)rem;
    }
    out->sched_len = (int64_t)sched.size();
    if ((int64_t)sched.size() > out->sched_cap || (!out->sched && !sched.empty()))
        return set_error(VIPER_E_INVAL, "sched_cap %lld < %lld needed", (long long)out->sched_cap,
                         (long long)sched.size());
    for (size_t k = 0; k < sched.size(); k++) out->sched[k] = sched[k];
    return VIPER_OK;
}
