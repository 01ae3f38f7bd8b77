"""oracle.selector -- TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

Simulation-based Selector of DTC-SpMM, step by step in the paper's order
(§4.5.2, Eq. (1), Fig. 10(b)/(c)), pure Python:

1. every row window w is one thread block of the base kernel, block_idx = w, whose
   length is its number of TC blocks RowWindowOffset[w+1] - RowWindowOffset[w];
2. Eq. (1): sm_idx = 2 (block_idx mod 64) + (floor(block_idx / 64) mod 2) on 128 SMs;
   for S SMs, 64 is read as S/2 (reading C23);
3. each SM runs `occupancy` blocks at once; the first `occupancy` blocks mapped to it
   start at time 0 and each later one starts when a resident block completes (the
   paper: "block 128 completes, the next block (block 768) is scheduled");
4. makespan = max over SMs of the last completion; with strict balance it is
   NumTCBlocks / (SMs x occupancy);
5. AR = makespan / balanced makespan; the balanced kernel is chosen when AR > 1.2.

Pinned by tests/test_selector.py (hand-worked schedules, uniform and single-window
closed forms, the paper's SM-0 example of Eq. (1)).
"""
from __future__ import annotations

import heapq

AR_THRESHOLD = 1.2


def eq1_sm(block_idx: int, num_sms: int = 128) -> int:
    """Eq. (1), PAPER.md:345 (C20 precedence), 64 = num_sms / 2."""
    half = num_sms // 2
    return 2 * (block_idx % half) + ((block_idx // half) % 2)


def makespan_base(rwo, num_sms: int = 128, occupancy: int = 6) -> int:
    lengths = [int(rwo[w + 1]) - int(rwo[w]) for w in range(len(rwo) - 1)]
    queues = [[] for _ in range(num_sms)]
    for b, length in enumerate(lengths):
        queues[eq1_sm(b, num_sms)].append(length)
    best = 0
    for q in queues:
        # resident slots as (finish time, slot index): the earliest finisher takes the next block
        slots = [(0, k) for k in range(occupancy)]
        heapq.heapify(slots)
        for length in q:
            t, k = heapq.heappop(slots)
            heapq.heappush(slots, (t + length, k))
        best = max(best, max(t for t, _ in slots))
    return best


def makespan_balanced(rwo, num_sms: int = 128, occupancy: int = 6) -> float:
    return (int(rwo[-1]) - int(rwo[0])) / (num_sms * occupancy)


def approximation_ratio(rwo, num_sms: int = 128, occupancy: int = 6) -> float:
    bal = makespan_balanced(rwo, num_sms, occupancy)
    return makespan_base(rwo, num_sms, occupancy) / bal if bal > 0 else 1.0


def select_balanced(rwo, num_sms: int = 128, occupancy: int = 6) -> bool:
    return approximation_ratio(rwo, num_sms, occupancy) > AR_THRESHOLD
