"""Test-side model of the paper's two-level stack and steal reservations, written
in the paper's notation but with this build's conventions: head/tail are monotone counters whose
slot is ``counter % hot_size`` (the kernel uses 16-bit counters), the flush moves the OLDEST
``batch`` entries from ``tail``, a refill fills the empty ring starting at ``tail``
(P:652-656), thieves reserve from ``tail`` / ``bottom`` (Alg 3 l.13-15, Alg 4 l.18-20).
The model reproduces the printed values of Figs 2 and 3 (tests/golden)."""
from __future__ import annotations


class HotRing:
    def __init__(self, hot_size: int, head: int = 0, tail: int = 0):
        self.hot_size = hot_size
        self.head, self.tail = head, tail              # slot = counter % hot_size
        self.slots = [None] * hot_size

    @property
    def hot_rest(self) -> int:                         # (head - tail + hot_size) % hot_size
        return (self.head - self.tail) % self.hot_size

    def full(self) -> bool:                            # (head + 1) % hot_size == tail
        return (self.head + 1) % self.hot_size == self.tail % self.hot_size

    def push(self, entry):                             # Fig 2(c)
        slot = self.head % self.hot_size
        self.slots[slot] = entry
        self.head = (self.head + 1) % self.hot_size
        return slot

    def pop(self):                                     # Fig 2(d)
        self.head = (self.head + self.hot_size - 1) % self.hot_size
        return self.head

    def flush(self, cold: "ColdSeg", batch: int):      # Fig 2(e): oldest `batch` entries from tail
        moved = []
        for q in range(batch):
            slot = (self.tail + q) % self.hot_size
            moved.append((slot, cold.top + q))
            cold.data[cold.top + q] = self.slots[slot]
        self.tail = (self.tail + batch) % self.hot_size
        cold.top += batch
        return moved

    def refill(self, cold: "ColdSeg", batch: int):     # Fig 2(f): from ColdSeg top into tail..
        k = min(batch, cold.top - cold.bottom)
        base = cold.top - k
        moved = []
        for q in range(k):
            slot = (self.tail + q) % self.hot_size
            self.slots[slot] = cold.data.get(base + q)
            moved.append((base + q, slot))
        self.head = (self.head + k) % self.hot_size
        cold.top -= k
        return moved


class ColdSeg:
    def __init__(self, top: int = 0, bottom: int = 0):
        self.top, self.bottom = top, bottom
        self.data = {}

    @property
    def cold_rest(self) -> int:
        return self.top - self.bottom


def intra_steal(rings, mask, thief, hot_cutoff):
    """Alg 3 for one idle warp; returns (victim or None).  Reservation = CAS on tail."""
    best, victim = 0, None
    for i, r in rings.items():                          # l.5-10
        if r.hot_rest > best:
            best, victim = r.hot_rest, i
    if victim is None or best < hot_cutoff:             # l.11
        return None
    hs = max(1, hot_cutoff // 2)                        # l.12
    v = rings[victim]
    old_tail = v.tail                                   # l.13-15 (CAS succeeds: no contention here)
    v.tail = (old_tail + hs) % v.hot_size
    t = rings[thief]
    for q in range(hs):                                 # l.17
        t.slots[(t.head + q) % t.hot_size] = v.slots[(old_tail + q) % v.hot_size]
    t.head = (t.head + hs) % t.hot_size                 # l.18
    mask[thief] = 1                                     # l.19
    return victim


def inter_steal(cold_segs, cold_cutoff):
    """Alg 4 steps 2-3 in the chosen victim block; returns (victim warp, reserved bottom)."""
    best, vw = 0, None
    for i, c in cold_segs.items():                      # l.9-15
        if c.cold_rest > best:
            best, vw = c.cold_rest, i
    if vw is None or best < cold_cutoff:                # l.16
        return None, None
    cs = max(1, cold_cutoff // 2)                       # l.17
    old = cold_segs[vw].bottom                          # l.18-20
    cold_segs[vw].bottom = old + cs
    return vw, old
