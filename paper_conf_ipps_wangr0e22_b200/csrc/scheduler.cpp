// scheduler.cpp — see scheduler.h.  Alg. 1 / Alg. 2 of PAPER.md, line numbers cited inline.
#include "scheduler.h"

#include <algorithm>

namespace micco {

Scheduler::Scheduler(int n_gpus, int policy, const int32_t bd[3], std::vector<int64_t> budget)
    : mem(n_gpus, 0), n(n_gpus), policy_(policy), budget_(std::move(budget)), count_(n_gpus, 0),
      com_(n_gpus, 0.0), com_total_(n_gpus, 0.0) {
  for (int i = 0; i < 3; ++i) bd_[i] = (policy == MICCO_POLICY_MICCO_NAIVE) ? 0 : bd[i];
}

void Scheduler::set_bounds(const int32_t bd[3]) {
  for (int i = 0; i < 3; ++i) bd_[i] = (policy_ == MICCO_POLICY_MICCO_NAIVE) ? 0 : bd[i];
}

void Scheduler::begin_vector(int64_t num_pairs) {
  balance_ = (num_pairs + n - 1) / n;  // balanceNum, reading #14
  std::fill(count_.begin(), count_.end(), 0);
  std::fill(com_.begin(), com_.end(), 0.0);
  rr_ = 0;
}

uint64_t Scheduler::candidates(const SchedPair &p) const {
  const uint64_t all = (n >= 64) ? ~0ULL : ((1ULL << n) - 1);
  uint64_t cand = 0;                                       // line 1
  const uint64_t g1 = p.m1, g2 = p.m2;                     // lines 2-3
  if (g1 & g2) {                                           // line 4: twoRepeatedSame
    for (uint64_t m = g1 & g2; m; m &= m - 1) {            // lines 5-6
      int g = __builtin_ctzll(m);
      if (count_[g] < bd_[0] + balance_) cand |= 1ULL << g;  // line 7
    }
  }
  if (!cand && (g1 | g2)) {                                // line 8 (∩ = AND, ∪ = OR, #11)
    for (uint64_t m = g1 | g2; m; m &= m - 1) {            // lines 9-14
      int g = __builtin_ctzll(m);
      if (count_[g] < bd_[1] + balance_) cand |= 1ULL << g;
    }
  }
  if (!cand) {                                             // line 15
    for (int g = 0; g < n; ++g)                            // line 16: all GPUs (#12)
      if (count_[g] < bd_[2] + balance_) cand |= 1ULL << g;  // lines 17-18
  }
  if (!cand) cand = all;                                   // reading #14 fallback
  return cand;
}

int64_t Scheduler::projected(int g, const SchedPair &p) const {  // reading #16
  int64_t m = mem[g];
  if (!((p.m1 >> g) & 1)) m += p.b1;
  if (!p.same && !((p.m2 >> g) & 1)) m += p.b2;
  if (p.b3 > 0 && !((p.m3 >> g) & 1)) m += p.b3;  // (the planner's need_bytes counts it too)
  return m + p.bout;
}

int Scheduler::assign(const SchedPair &p, uint64_t cand) const {
  bool evict = false;                                      // Alg. 2 lines 1-5
  for (uint64_t m = cand; m; m &= m - 1) {
    int g = __builtin_ctzll(m);
    if (projected(g, p) > budget_[g]) evict = true;
  }
  // MICCO_AFFINITY (p.pref >= 0 only under that policy): the last consumer's GPU, if Alg. 1
  // admitted it and no oversubscription is projected
  if (!evict && p.pref >= 0 && ((cand >> p.pref) & 1)) return p.pref;
  int best = -1;
  for (uint64_t m = cand; m; m &= m - 1) {
    int g = __builtin_ctzll(m);
    if (best < 0) { best = g; continue; }
    if (!evict) {  // lines 6-11: least computation, ties least memory, then id (#17)
      if (com_[g] < com_[best] || (com_[g] == com_[best] && mem[g] < mem[best])) best = g;
    } else {       // lines 12-17: most available memory, ties least computation, then id
      const int64_t fg = budget_[g] - mem[g], fb = budget_[best] - mem[best];
      if (fg > fb || (fg == fb && com_[g] < com_[best])) best = g;
    }
  }
  return best;                                             // line 18
}

int Scheduler::decide(const SchedPair &p) {
  switch (policy_) {
    case MICCO_POLICY_ROUND_ROBIN:
      return (int)(rr_++ % n);
    case MICCO_POLICY_LEAST_LOADED: {  // earliest-available device (Groute rule, L312)
      int best = 0;
      for (int g = 1; g < n; ++g)
        if (com_total_[g] < com_total_[best]) best = g;
      return best;
    }
    default:
      return assign(p, candidates(p));                     // Alg. 1 line 19
  }
}

void Scheduler::account(int g, const SchedPair &p) {       // Alg. 1 line 20 (non-residency part)
  ++count_[g];
  com_[g] += p.flops;
  com_total_[g] += p.flops;
}

}  // namespace micco
