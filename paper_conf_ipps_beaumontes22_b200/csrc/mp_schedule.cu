// mp_schedule.cu -- NEXT row f2: the 1F1B* periodic pattern of a contiguous
// allocation (Section 4.1 of the paper), as a host-only C ABI entry.
//
// Given stages s_1..s_N (contiguous, one per GPU) and a period T:
//   * the comm -> layer transform: between consecutive stages the
//     activation a^(l) (forward) and the gradient b^(l) (backward) cross the
//     link, each taking a_l / beta, so the chain of N stages becomes a chain of
//     2N-1 communication-free items with loads U(s) and C(l) = 2 a_l / beta;
//   * groups: from the last item backwards, add items while the group's
//     total load stays <= T; group 1 holds the last item;
//   * pattern: forward operations of all items in sequence with index
//     shift 0; each group's backward operations start right after its last
//     forward operation, in reverse order, with shift g-1; finally every start
//     time >= T is lowered by T and its shift increased by 1.
// Every item of group g keeps exactly g activations alive (Proposition 1).
// This is product code: it shares nothing with oracle/simulator.py, which the
// tests use to check it.
#include <cmath>
#include <cstdint>
#include <vector>

#include "../../include/madpipe.h"

extern "C" int madpipe_schedule(const madpipe_chain *chain, double beta, double period, int32_t n_stages,
                                const int32_t *stage_first, const int32_t *stage_last, madpipe_op *ops,
                                int32_t *n_ops) {
    if (!chain || !stage_first || !stage_last || !ops || !n_ops || n_stages < 1 || !(period > 0.0) ||
        !(beta > 0.0))
        return MADPIPE_EINVAL;
    const int L = chain->L;
    // stages must tile 1..L in order
    int pos = 1;
    for (int s = 0; s < n_stages; s++) {
        if (stage_first[s] != pos || stage_last[s] < stage_first[s] || stage_last[s] > L) return MADPIPE_EINVAL;
        pos = stage_last[s] + 1;
    }
    if (pos != L + 1) return MADPIPE_EINVAL;
    const int n = 2 * n_stages - 1;
    std::vector<double> uf(n), ub(n);
    std::vector<int> kind(n), index(n);
    for (int s = 0, it = 0; s < n_stages; s++) {
        if (s > 0) {   // communication of a^(l) / b^(l), l = first layer of s minus 1
            const double c = (double)chain->a[stage_first[s] - 1] / beta;
            uf[it] = c; ub[it] = c; kind[it] = 1; index[it] = s; it++;
        }
        double f = 0.0, b = 0.0;
        for (int i = stage_first[s]; i <= stage_last[s]; i++) {
            f += chain->uF[i - 1];
            b += chain->uB[i - 1];
        }
        uf[it] = f; ub[it] = b; kind[it] = 0; index[it] = s; it++;
    }
    for (int i = 0; i < n; i++)
        if (uf[i] + ub[i] > period) return MADPIPE_INFEASIBLE;   // an item longer than the period
    // groups, from the end
    std::vector<int> group(n);
    int g = 1;
    double acc = 0.0;
    for (int i = n - 1; i >= 0; i--) {
        const double u = uf[i] + ub[i];
        if (acc > 0.0 && acc + u > period) { g++; acc = 0.0; }
        acc += u;
        group[i] = g;
    }
    // forward chain with shift 0, backward per group after its last forward
    std::vector<double> tf(n), tb(n);
    std::vector<int> hb(n);
    double t = 0.0;
    for (int i = 0; i < n; i++) { tf[i] = t; t += uf[i]; }
    for (int j = n - 1; j >= 0;) {
        int first = j;
        while (first - 1 >= 0 && group[first - 1] == group[j]) first--;
        double tb0 = tf[j] + uf[j];
        for (int q = j; q >= first; q--) { tb[q] = tb0; hb[q] = group[j] - 1; tb0 += ub[q]; }
        j = first - 1;
    }
    for (int i = 0; i < n; i++) {
        madpipe_op &o = ops[i];
        o.kind = kind[i];
        o.stage = index[i];
        o.group = group[i];
        double f = tf[i], b = tb[i];
        int hf = 0, h = hb[i];
        while (f >= period) { f -= period; hf++; }
        while (b >= period) { b -= period; h++; }
        o.f_start = f; o.f_shift = hf; o.f_len = uf[i];
        o.b_start = b; o.b_shift = h; o.b_len = ub[i];
    }
    *n_ops = n;
    return MADPIPE_OK;
}
