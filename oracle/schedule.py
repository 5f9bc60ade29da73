"""Oracle of the advance-forward-propagation micro-batch order (Algorithm 1).

TEST INFRASTRUCTURE ONLY -- see ``oracle/__init__.py``.

Paper (§4):
  P:124-130  AFAB: all forwards of a batch, then all backwards (Fig. 7(a)).
  P:132      1F1B: alternate forward and backward; with K GPUs "the k-th GPU
             only needs to stash the activation of up to K-k+1 micro-batches";
             K=2, k=1 stashes 2 (Fig. 7(b)).
  P:140-157  Algorithm 1, on the 1st GPU: run ``advance_num`` forwards, then
             M - advance_num times (forward, backward).  Line 1 starts at
             advance_num = K - 1, "equivalent to 1F1B".
  P:164-168  advance forward stashes 3 micro-batches on GPU 1 in Fig. 7(c)
             (1F1B: 2) and peaks at 3/8 of AFAB; it degenerates to 1F1B
             (fewest advances) or AFAB ("all micro-batches in advance").

Readings (DESIGN.md c15/c16/c19):
  c15  Algorithm 1 omits the cool-down: after the interleaved loop the
       backwards of the remaining advance_num micro-batches follow in order.
       advance_num is clamped to [0, M] (M = AFAB).  For GPU k
       (1-based) the 1F1B starting point is K-k; micro-batch ids are 0-based.
  c19  Fig. 7's M is not printed; "3 of AFAB's 8" implies M = 8.

Ops are ('F', j) / ('B', j) tuples.
"""
from __future__ import annotations

from typing import Dict, List, Sequence, Tuple

Op = Tuple[str, int]


def advance_forward_schedule(K: int, M: int, k: int, advance_num: int) -> List[Op]:
    """Op order of GPU k (1-based, 1 <= k <= K) for one batch of M micro-batches
    with ``advance_num`` forwards in advance (Algorithm 1 + c15 cool-down)."""
    if K < 1 or M < 0 or not (1 <= k <= K):
        raise ValueError("need K >= 1, M >= 0, 1 <= k <= K")
    a = min(max(advance_num, 0), M)
    ops: List[Op] = []
    f = 0   # next micro-batch to forward
    b = 0   # next micro-batch to backward
    for _ in range(a):                # Alg. 1 lines 3-4: forward in advance
        ops.append(("F", f)); f += 1
    for _ in range(M - a):            # Alg. 1 lines 6-8: interleave the rest
        ops.append(("F", f)); f += 1
        ops.append(("B", b)); b += 1
    while b < M:                      # c15: cool-down (implied)
        ops.append(("B", b)); b += 1
    return ops


def one_f_one_b_advance(K: int, k: int) -> int:
    """1F1B as the advance count K - k (Alg. 1 line 1 for k = 1)."""
    return K - k


def default_advance(K: int, M: int, k: int, extra: int = 0) -> int:
    """c15: per-GPU advance a_k = min(M, K - k + extra); extra = 0 is 1F1B."""
    return min(M, K - k + extra)


def peak_in_flight(ops: Sequence[Op]) -> int:
    """Maximum number of micro-batches whose forward ran but whose backward has
    not (the activation stash the schedule implies)."""
    live = peak = 0
    for kind, _ in ops:
        live += 1 if kind == "F" else -1
        peak = max(peak, live)
    return peak


def simulate_pipeline(K: int, M: int, advances: Sequence[int]) -> Dict[str, object]:
    """Brute-force check that per-GPU op lists can run together (reading c16).

    GPU k executes its list in order; F(k, j) needs F(k-1, j) done, B(k, j)
    needs B(k+1, j) done (sends are asynchronous and unbounded).  Repeatedly
    run any GPU whose next op is ready; deadlock if none can move.
    Returns {"ok": bool, "order": [(k, op), ...]}.
    """
    lists = [advance_forward_schedule(K, M, k, advances[k - 1]) for k in range(1, K + 1)]
    pos = [0] * K
    done = set()
    order = []
    progressed = True
    while progressed:
        progressed = False
        for k in range(1, K + 1):
            if pos[k - 1] >= len(lists[k - 1]):
                continue
            kind, j = lists[k - 1][pos[k - 1]]
            if kind == "F":
                ready = k == 1 or (k - 1, "F", j) in done
            else:
                ready = (k, "F", j) in done and (k == K or (k + 1, "B", j) in done)
            if ready:
                done.add((k, kind, j))
                order.append((k, (kind, j)))
                pos[k - 1] += 1
                progressed = True
    ok = all(pos[k] == len(lists[k]) for k in range(K))
    return {"ok": ok, "order": order}


class AdvanceController:
    """Algorithm 1's run-time adjustment of ``advance_num``.

    Line 1: advance_num <- K - 1 (1F1B on GPU 1).  After every batch (lines
    9-10): if is_faster() and is_mem_available() then advance_num++.

    Readings (DESIGN.md c27):
      is_faster()        the batch just finished took strictly less time than
                         the batch before it; the first batch has nothing to
                         compare with and counts as faster (exploration starts).
      is_mem_available() peak memory of the batch + the activation stash of one
                         more micro-batch <= the user's limit (one more forward
                         in advance holds one more micro-batch).
      advance_num never exceeds M (AFAB) and never decreases.
      GPU k (1-based) runs min(M, K - k + extra) with extra = advance_num - (K-1) (c15).
    """

    def __init__(self, K: int, M: int):
        if K < 1 or M < 0:
            raise ValueError("need K >= 1 and M >= 0")
        self.K, self.M = K, M
        self.advance_num = min(K - 1, M)      # Alg. 1 line 1
        self.last_time = None

    def is_faster(self, batch_time: float) -> bool:
        return self.last_time is None or batch_time < self.last_time

    @staticmethod
    def is_mem_available(peak_mem: float, mem_per_microbatch: float, mem_limit: float) -> bool:
        return peak_mem + mem_per_microbatch <= mem_limit

    def update(self, batch_time: float, peak_mem: float, mem_per_microbatch: float, mem_limit: float) -> int:
        """Lines 9-10 after one batch; returns the advance_num for the next batch."""
        if self.is_faster(batch_time) and self.is_mem_available(peak_mem, mem_per_microbatch, mem_limit):
            if self.advance_num < self.M:
                self.advance_num += 1
        self.last_time = batch_time
        return self.advance_num

    def advance_for(self, k: int) -> int:
        """advance of GPU k (1-based)."""
        extra = self.advance_num - min(self.K - 1, self.M)
        return default_advance(self.K, self.M, k, extra)
