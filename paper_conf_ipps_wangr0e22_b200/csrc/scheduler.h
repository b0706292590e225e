// scheduler.h — MICCO's heuristic scheduling algorithm (§IV-B, Alg. 1 + Alg. 2,
// L195-288) and the baseline policies, as one decision function shared by the planner and
// the micco_debug_schedule test hook.
//
// State follows Table III (L179-193) with the SURVEY.md §8(c) readings:
//   residency mask per tensor (mapGPUTensor.find, #13), count[g] = pairs assigned to g in the
//   current vector (mapGPUTensor.at(g).size(), #13/#15), com[g] = flops assigned in the current
//   vector (mapGPUCom, #18), mem[g] = bytes resident (mapGPUMem), budget[g] (GPUMaxMemory),
//   balanceNum = ceil(numPairs / numGPU) (#14); ties broken lexicographically (#17).
#pragma once

#include <cstdint>
#include <vector>

#include "micco.h"

namespace micco {

struct SchedPair {
  uint64_t m1, m2;            // residency masks of Tensor1, Tensor2 (bit g = resident on GPU g)
  bool same;                  // Tensor1 == Tensor2
  int64_t b1, b2, bout;       // bytes
  uint64_t m3 = 0;            // a third operand read by the task (the fused final dot's partner)
  int64_t b3 = 0;             // ... and its bytes (0 = none)
  double flops;
  int pref = -1;              // MICCO_AFFINITY: GPU of the operands' last consumer (-1 = none)
};

class Scheduler {
 public:
  Scheduler(int n_gpus, int policy, const int32_t bd[3], std::vector<int64_t> budget);
  void begin_vector(int64_t num_pairs);
  // Alg. 1 lines 1-18: candidate mask
  uint64_t candidates(const SchedPair &p) const;
  // Alg. 2: choose among candidates (projected-memory eviction test, then min computation or
  // min memory)
  int assign(const SchedPair &p, uint64_t cand) const;
  // the full decision for one pair under the configured policy
  int decide(const SchedPair &p);
  // line 20 bookkeeping that is not residency: count, com (and cumulative load)
  void account(int g, const SchedPair &p);
  // reuseBd for the next vectors (per-vector bounds)
  void set_bounds(const int32_t bd[3]);
  std::vector<int64_t> mem;   // mapGPUMem, maintained by the caller
  int n;
 private:
  int policy_;
  int32_t bd_[3];
  std::vector<int64_t> budget_;
  std::vector<int64_t> count_;
  std::vector<double> com_, com_total_;
  int64_t balance_ = 0;
  int64_t rr_ = 0;
  int64_t projected(int g, const SchedPair &p) const;
};

}  // namespace micco
