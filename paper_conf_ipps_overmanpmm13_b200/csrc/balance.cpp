// balance.cpp -- load-balancing state machine (include/afmm_balance.h).
// PAPER.md L18 SV (states), L20 SVI-SVII (Enforce_S, FineGrainedOptimize, timing,
// state switching), L22 (the 5% observation rule).
#include <algorithm>
#include <cmath>
#include <new>

#include "../../include/afmm_balance.h"

struct afmm_lb {
    afmm_lb_config cfg{};
    int state = AFMM_LB_SEARCH;
    int S = 128;
    int lo = 1, hi = 1;            // SEARCH bracket
    int dominant = 0;              // INCREMENTAL: +1 CPU dominates, -1 GPU dominates, 0 unset
    double best = 0.0;             // OBSERVATION: best compute time
    bool rebest = false;           // next measured compute time becomes the best (after Enforce_S)
    int pending = AFMM_LB_KEEP;    // ENFORCE / FINE awaiting a predicted time
    bool to_incremental = false;   // fine-grained adjustment failed: INCREMENTAL next step
    bool fine_from_incremental = false;
};

extern "C" afmm_status afmm_lb_config_init(afmm_lb_config *c) {
    if (!c) return AFMM_EINVAL;
    c->S_init = 128;
    c->S_min = 8;
    c->S_max = 2048;
    c->dS = 8;
    c->balance_rel = 0.15;
    c->observe_rel = 0.05;
    return AFMM_OK;
}

extern "C" afmm_status afmm_lb_create(const afmm_lb_config *c, afmm_lb **out) {
    if (!out) return AFMM_EINVAL;
    *out = nullptr;
    if (!c || c->S_min < 1 || c->S_min > c->S_init || c->S_init > c->S_max || c->dS < 1 ||
        !(c->balance_rel > 0.0) || !(c->observe_rel > 0.0) || !std::isfinite(c->balance_rel) ||
        !std::isfinite(c->observe_rel))
        return AFMM_EINVAL;
    afmm_lb *lb = new (std::nothrow) afmm_lb();
    if (!lb) return AFMM_ENOMEM;
    lb->cfg = *c;
    lb->S = c->S_init;
    lb->lo = c->S_min;
    lb->hi = c->S_max;
    *out = lb;
    return AFMM_OK;
}

extern "C" void afmm_lb_destroy(afmm_lb *lb) { delete lb; }

extern "C" afmm_status afmm_lb_state(const afmm_lb *lb, int *state, int *S, double *best) {
    if (!lb) return AFMM_EINVAL;
    if (state) *state = lb->state;
    if (S) *S = lb->S;
    if (best) *best = lb->best;
    return AFMM_OK;
}

static void enter_observation(afmm_lb *lb, double compute) {
    lb->state = AFMM_LB_OBSERVATION;
    lb->best = compute;                       // "the current compute time ... is recorded"
    lb->rebest = false;
}

extern "C" afmm_status afmm_lb_step(afmm_lb *lb, double t_cpu, double t_gpu, int *action, int *S) {
    if (!lb || !action || !S) return AFMM_EINVAL;
    if (!(t_cpu >= 0.0) || !(t_gpu >= 0.0) || !std::isfinite(t_cpu) || !std::isfinite(t_gpu)) return AFMM_EINVAL;
    if (lb->pending != AFMM_LB_KEEP) return AFMM_ESTATE;
    const afmm_lb_config &c = lb->cfg;
    const double compute = std::max(t_cpu, t_gpu);                   // L20 SVII.A
    const bool balanced = std::fabs(t_cpu - t_gpu) <= c.balance_rel * compute;
    const int dom = t_cpu > t_gpu ? 1 : (t_gpu > t_cpu ? -1 : 0);
    *action = AFMM_LB_KEEP;
    if (lb->to_incremental) {                 // the fine-grained adjustment failed last step
        lb->to_incremental = false;
        lb->state = AFMM_LB_INCREMENTAL;
        lb->dominant = 0;
    }
    switch (lb->state) {
    case AFMM_LB_SEARCH: {
        if (balanced || lb->hi - lb->lo <= 1) {
            lb->state = AFMM_LB_INCREMENTAL;
            lb->dominant = 0;
            // fall through to the incremental rule on this step's times
        } else {
            // larger S moves work from the far field (CPU) to the near field (GPU), L14 SIII.A
            if (dom > 0) lb->lo = lb->S;
            else lb->hi = lb->S;
            const int next = lb->lo + (lb->hi - lb->lo) / 2;
            if (next == lb->S) {
                lb->state = AFMM_LB_INCREMENTAL;
                lb->dominant = 0;
            } else {
                lb->S = next;
                *action = AFMM_LB_REBUILD;
                break;
            }
        }
    }
    // fallthrough
    case AFMM_LB_INCREMENTAL: {
        if (lb->state != AFMM_LB_INCREMENTAL) break;
        if (lb->dominant == 0) lb->dominant = dom == 0 ? 1 : dom;
        if (dom != 0 && dom != lb->dominant) {                          // the transitional S
            if (!balanced) {                  // FineGrainedOptimize, then OBSERVATION in any case
                lb->pending = AFMM_LB_FINE;
                lb->fine_from_incremental = true;
                lb->state = AFMM_LB_OBSERVATION;
                lb->best = compute;
                *action = AFMM_LB_FINE;
            } else {
                enter_observation(lb, compute);
            }
            break;
        }
        const int next = std::min(c.S_max, std::max(c.S_min, lb->S + (lb->dominant > 0 ? c.dS : -c.dS)));
        if (next == lb->S) {                                             // bracket edge: settle
            enter_observation(lb, compute);
        } else {
            lb->S = next;
            *action = AFMM_LB_REBUILD;
        }
        break;
    }
    case AFMM_LB_OBSERVATION: {
        if (lb->rebest) {                     // "the compute time on the time step immediately following
            lb->best = compute;               //  Enforce_S() calls becomes the new best time"
            lb->rebest = false;
            break;
        }
        if (compute > lb->best * (1.0 + c.observe_rel)) {
            lb->fine_from_incremental = false;
            lb->pending = AFMM_LB_ENFORCE;
            *action = AFMM_LB_ENFORCE;
        }                                     // else "nothing is done" (L22): the best stays as recorded
        break;
    }
    }
    *S = lb->S;
    return AFMM_OK;
}

extern "C" afmm_status afmm_lb_predicted(afmm_lb *lb, double t_pred, int *action) {
    if (!lb || !action) return AFMM_EINVAL;
    if (!(t_pred >= 0.0) || !std::isfinite(t_pred)) return AFMM_EINVAL;
    if (lb->pending == AFMM_LB_KEEP) return AFMM_ESTATE;
    const bool ok = t_pred <= lb->best * (1.0 + lb->cfg.observe_rel);
    *action = AFMM_LB_KEEP;
    if (lb->pending == AFMM_LB_ENFORCE) {
        if (ok) {
            lb->pending = AFMM_LB_KEEP;
            lb->rebest = true;
        } else {
            lb->pending = AFMM_LB_FINE;
            *action = AFMM_LB_FINE;
        }
    } else {                                   // after FineGrainedOptimize
        lb->pending = AFMM_LB_KEEP;
        if (lb->fine_from_incremental) {       // at the transitional S: "upon return from this function the load
            lb->fine_from_incremental = false; //  balancer enters the observation state" with the best recorded
        } else if (ok) {                       //  before it (L20 SVII.B)
            lb->rebest = true;                 // after Enforce_S: the next step's compute time is the best (L24-L26)
        } else {
            lb->to_incremental = true;         // "moves into the incremental state again on the following time step"
        }
    }
    return AFMM_OK;
}

extern "C" afmm_status afmm_lb_predict(const long long *counts, const double *coef, double *t_cpu, double *t_gpu,
                                       double *t) {
    if (!counts || !coef) return AFMM_EINVAL;
    for (int i = 0; i < 6; ++i)
        if (counts[i] < 0 || !(coef[i] >= 0.0) || !std::isfinite(coef[i])) return AFMM_EINVAL;
    double cpu = 0.0;
    for (int i = 0; i < 5; ++i) cpu += coef[i] * (double)counts[i];       // T_cpu = sum_op C_op M(op)
    const double gpu = coef[5] * (double)counts[5];                       // T_gpu = C_P2P M(P2P)
    if (t_cpu) *t_cpu = cpu;
    if (t_gpu) *t_gpu = gpu;
    if (t) *t = std::max(cpu, gpu);                                       // compute time (L20 SVII.A)
    return AFMM_OK;
}
