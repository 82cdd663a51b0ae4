"""Algorithm 1 with contention factor and runtime decomposition (oracle; test infra only).

PAPER.md §3.3-3.6.  One scheduling round, with the readings listed
in DESIGN.md (R1 comparator swap, R2 list-end switch, R3 cf placement, R5
largest-fitting piece, R6/R7 what is decomposable and how):

 (1) update_list(): remove finished batches from the processing list and admit
     from the waiting queue, FIFO by arrival, up to the list size.
 (2) Primary subset: pop kernels of FuncVec[0] into SubSet0, accumulating
     time += dur, up to and including the kernel whose successor has the other
     type, or the end of the list (switch point P:170).
     type := type of that last kernel.
 (3) For V in FuncVec[1:] (arrival order): while time > 0 and V non-empty and
     V.front.type != type:
       if cf*dur(V.front) <= time: push it to SubSet1, time -= cf*dur
                                   (the printed comparator is inverted, R1;
                                    cf scales the secondary durations)
       elif V.front is decomposable (GEMM / all-reduce) and has > 1
            unit left: push the largest k/F piece with cf*dur(k/F) <= time,
            leave the remainder at the head; if none fits,
            time = 0
       else: time = 0
     If V.front has the same type as the primary subset, move to the next V.
 (4) SubSet1 and SubSet0 are launched on the streams of their types, the
     communication subset first.

Kernel durations are profiled per (kernel, k/F); `durs[k-1]` is
the duration of a k-unit piece.  A non-decomposable kernel has one unit.
"""
from collections import deque
from dataclasses import dataclass, field


@dataclass
class Kernel:
    batch: int
    name: str
    type: str                  # "C" (computation) or "M" (communication)
    durs: tuple                # durs[k-1] = profiled duration of a k-unit piece
    decomposable: bool = False
    done: int = 0              # units already launched

    @property
    def units(self):
        return len(self.durs)

    @property
    def left(self):
        return self.units - self.done

    def dur_of(self, k):
        return self.durs[k - 1]

    @property
    def dur_left(self):
        return self.dur_of(self.left)


@dataclass
class Piece:
    batch: int
    name: str
    type: str
    u0: int      # first unit (inclusive)
    u1: int      # last unit (exclusive)
    units: int   # total units of the kernel
    dur: float   # profiled duration of this piece (unscaled)


@dataclass
class Round:
    sub0: list = field(default_factory=list)
    sub1: list = field(default_factory=list)
    type: str = "C"
    time0: float = 0.0       # sum of SubSet0 durations
    time1_scaled: float = 0.0  # cf * sum of SubSet1 durations


def _take(k: Kernel, n: int) -> Piece:
    p = Piece(k.batch, k.name, k.type, k.done, k.done + n, k.units, k.dur_of(n))
    k.done += n
    return p


def plan_round(flists, cf=1.0):
    """One iteration of Algorithm 1 over the processing list `flists`
    (list of deques of Kernel, index 0 = primary = earliest batch)."""
    r = Round()
    prim = flists[0]
    time = 0.0
    typ = None
    while prim:
        k = prim[0]
        time += k.dur_left
        typ = k.type
        r.sub0.append(_take(k, k.left))
        prim.popleft()
        if not prim or prim[0].type != typ:      # switch point (or list end, R2)
            break
    r.type = typ
    r.time0 = time
    for V in flists[1:]:
        while time > 0 and V and V[0].type != typ:
            k = V[0]
            c = cf * k.dur_left
            if c <= time:
                r.sub1.append(_take(k, k.left))
                V.popleft()
                time -= c
                r.time1_scaled += c
            elif k.decomposable and k.left > 1:
                best = 0
                for n in range(1, k.left):
                    if cf * k.dur_of(n) <= time:
                        best = n
                if best == 0:
                    time = 0.0
                else:
                    c = cf * k.dur_of(best)
                    r.sub1.append(_take(k, best))
                    time -= c
                    r.time1_scaled += c
            else:
                time = 0.0
        if time <= 0:
            break
    return r


class Scheduler:
    """Waiting queue + fixed-size processing list (Fig. 7) driving plan_round."""

    def __init__(self, list_size=2, cf=1.0):
        self.list_size = list_size
        self.cf = cf
        self.waiting = deque()
        self.processing = []     # list of (batch_id, deque[Kernel])

    def submit(self, batch_id, kernels):
        self.waiting.append((batch_id, deque(kernels)))

    def update_list(self):
        self.processing = [(b, q) for (b, q) in self.processing if q]
        while len(self.processing) < self.list_size and self.waiting:
            self.processing.append(self.waiting.popleft())

    def step(self):
        self.update_list()
        if not self.processing:
            return None
        return plan_round([q for _, q in self.processing], self.cf)

    def run(self):
        rounds = []
        while True:
            r = self.step()
            if r is None:
                return rounds
            rounds.append(r)
