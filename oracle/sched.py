"""Scheduler oracle — MICCO's heuristic scheduling algorithm restated line by
line from the paper (test infrastructure only; see oracle/__init__.py).

Alg. 1 (steps I-IV L248-252) builds ``candiQueue`` for one
tensor pair; Alg. 2 (L254-288) picks the GPU.  Variables follow Table III
(L179-193).  Where the extracted pseudo-code is garbled or ambiguous the
SURVEY.md §8(c) readings are taken, each cited inline:

* #11  ``∩``/``∪`` in the conditions of Alg. 1 are logical AND / OR.
* #12  line 16 ``for it = 1; it < numGPU`` scans ALL GPUs 0..numGPU-1.
* #13  ``mapGPUTensor`` is two structures: residency (tensor → set of GPUs)
       and the per-vector count of pairs per GPU (``.at(g).size()``).
* #14  balanceNum = ceil(numPairs / numGPU); if candiQueue is still empty
       after line 18, every GPU is a candidate.
* #15  counts are tensor PAIRS per GPU per vector.
* #16  the oversubscription test of Alg. 2 line 4 uses PROJECTED bytes:
       resident + operand copies this pair needs + its output.
* #17  ``random(min(...))`` ties are broken deterministically:
       (computation, memory, gpu id) normally, (memory, computation, gpu id)
       in eviction mode.
* #18  mapGPUCom is the flops assigned to the GPU in the current vector.

The update of line 20 makes both operands and the output resident on the
chosen GPU.  This oracle models no eviction (the memory test only selects the
policy), so it is compared with the native scheduler decision for decision
under budgets where nothing is evicted; under pressure the native planner is
checked by invariants instead (tests/test_scheduler.py).
"""
from __future__ import annotations

import math
from dataclasses import dataclass
from typing import Dict, List, Sequence, Set

TWO_REPEATED_SAME, TWO_REPEATED_DIFF, ONE_REPEATED, TWO_NEW = 0, 1, 2, 3


@dataclass
class Pair:
    t1: int          # operand tensor ids (Tensor1, Tensor2 of Table III)
    t2: int
    out: int         # id of the produced tensor
    flops: float     # computation cost of the contraction
    b1: int          # bytes of Tensor1, Tensor2, output
    b2: int
    bout: int


def local_reuse_pattern(res: Dict[int, Set[int]], t1: int, t2: int) -> int:
    """Fig. 4 / L126-132: twoRepeatedSame, twoRepeatedDiff, oneRepeated, twoNew."""
    g1, g2 = res.get(t1, set()), res.get(t2, set())
    if g1 & g2:
        return TWO_REPEATED_SAME
    if g1 and g2:
        return TWO_REPEATED_DIFF
    if g1 or g2:
        return ONE_REPEATED
    return TWO_NEW


class MiccoSchedulerOracle:
    def __init__(self, num_gpu: int, reuse_bd: Sequence[int], gpu_max_memory: float):
        self.num_gpu = num_gpu
        self.reuse_bd = list(reuse_bd)
        self.gpu_max_memory = gpu_max_memory
        self.res: Dict[int, Set[int]] = {}          # mapGPUTensor, residency part (#13)
        self.mem = [0] * num_gpu                     # mapGPUMem (bytes resident)
        self.count = [0] * num_gpu                   # mapGPUTensor.at(g).size() (#13, #15)
        self.com = [0.0] * num_gpu                   # mapGPUCom (#18)
        self.balance_num = 0

    def begin_vector(self, num_pairs: int):
        self.balance_num = math.ceil(num_pairs / self.num_gpu)   # #14
        self.count = [0] * self.num_gpu
        self.com = [0.0] * self.num_gpu

    # ---- Alg. 1 lines 1-18
    def candidates(self, p: Pair) -> List[int]:
        bd, bal = self.reuse_bd, self.balance_num
        cand: List[int] = []                                          # line 1
        g1 = sorted(self.res.get(p.t1, set()))                        # line 2
        g2 = sorted(self.res.get(p.t2, set()))                        # line 3
        if set(g1) & set(g2):                                         # line 4
            for it1 in g1:                                            # line 5
                if it1 in g2 and self.count[it1] < bd[0] + bal:       # line 6 (#11)
                    cand.append(it1)                                  # line 7
        if not cand and (g1 or g2):                                   # line 8 (#11)
            for it1 in g1:                                            # line 9
                if self.count[it1] < bd[1] + bal:                     # line 10
                    cand.append(it1)                                  # line 11
            for it2 in g2:                                            # line 12
                if self.count[it2] < bd[1] + bal and it2 not in cand:  # line 13
                    cand.append(it2)                                  # line 14
        if not cand:                                                  # line 15
            for it in range(self.num_gpu):                            # line 16 (#12)
                if self.count[it] < bd[2] + bal:                      # line 17
                    cand.append(it)                                   # line 18
        if not cand:                                                  # #14 fallback
            cand = list(range(self.num_gpu))
        return cand

    def projected_mem(self, g: int, p: Pair) -> int:                 # #16
        m = self.mem[g]
        if g not in self.res.get(p.t1, set()):
            m += p.b1
        if p.t2 != p.t1 and g not in self.res.get(p.t2, set()):
            m += p.b2
        return m + p.bout

    # ---- Alg. 2
    def assign(self, p: Pair, cand: List[int]) -> int:
        evict = any(self.projected_mem(g, p) > self.gpu_max_memory for g in cand)   # lines 3-5
        if not evict:                                                               # line 6
            return min(cand, key=lambda g: (self.com[g], self.mem[g], g))           # lines 7-11 (#17)
        return min(cand, key=lambda g: (self.mem[g], self.com[g], g))               # lines 12-17 (#17)

    def schedule(self, p: Pair) -> int:
        g = self.assign(p, self.candidates(p))                       # line 19
        # line 20: update mapGPUTensor, mapGPUCom, mapGPUMem
        for t, b in ((p.t1, p.b1), (p.t2, p.b2)):
            s = self.res.setdefault(t, set())
            if g not in s:
                s.add(g)
                self.mem[g] += b
        self.res.setdefault(p.out, set()).add(g)
        self.mem[g] += p.bout
        self.count[g] += 1
        self.com[g] += p.flops
        return g                                                      # line 21

    def run(self, vectors: Sequence[Sequence[Pair]]) -> List[List[int]]:
        out = []
        for vec in vectors:
            self.begin_vector(len(vec))
            out.append([self.schedule(p) for p in vec])
        return out
