"""Host model of the device-initiated multi-GPU protocol (csrc/kcore_mgd.cu),
test infrastructure only (SURVEY 8(c) tier T4: "the host model of the mg
protocol (P=1..8) vs oracle").  Each rank owns a vertex range and its rows;
every step below mirrors one phase of the kernel:

  init   deg = degree, isolated vertices removed (deg += REMOVED), core 0
  scan   own alive vertices with deg <= k: removed, core k, into own inbox;
         min over deg > k (level skip, reading R5)
  peel   every rank walks the rows of its inbox; each arc's decrement is a
         message to the target's owner (the kernel's remote atomicSub), which
         applies it and appends the target to its next inbox when the old
         value was k+1; old > k+1 feeds the minimum
  level  ends when a sub-round pushed nothing; k <- max(k+1, global min)

The exchange of decrement messages and the global reductions are callbacks,
so the same rank code runs with P in-process ranks or with one rank per
torch.distributed process (gloo).  It shares no code with the oracle."""
import numpy as np

REMOVED = 1 << 30
DEAD = 1 << 29


class Rank:
    def __init__(self, rp_local, ci_local, vb, ve, ranges):
        self.rp = np.asarray(rp_local, dtype=np.int64)
        self.ci = np.asarray(ci_local, dtype=np.int64)
        self.vb, self.ve = vb, ve
        self.ranges = ranges
        self.starts = np.array([a for a, _ in ranges], dtype=np.int64)
        nl = ve - vb
        d = np.diff(self.rp)
        self.deg = np.where(d > 0, d, REMOVED).astype(np.int64)
        self.core = np.full(nl, -1, dtype=np.int64)
        self.core[d == 0] = 0
        self.inbox = []
        self.next_inbox = []

    def init_stats(self):
        d = np.diff(self.rp)
        pos = d[d > 0]
        return int((d == 0).sum()), (int(pos.min()) if pos.size else None)

    def owner(self, u):
        return np.searchsorted(self.starts, u, side="right") - 1

    def scan(self, k):
        alive = self.deg < DEAD
        fr = np.nonzero(alive & (self.deg <= k))[0]
        self.deg[fr] += REMOVED
        self.core[fr] = k
        self.inbox = list(fr)
        rest = self.deg[alive & (self.deg > k)]
        return len(fr), (int(rest.min()) if rest.size else None)

    def walk(self, k):
        """Messages {owner: [local target ids]} for every arc of the inbox rows."""
        msgs = {}
        for v in self.inbox:
            self.core[v] = k
            tg = self.ci[self.rp[v]:self.rp[v + 1]]
            own = self.owner(tg)
            for o in np.unique(own):
                msgs.setdefault(int(o), []).extend((tg[own == o] - self.ranges[o][0]).tolist())
        self.inbox = []
        return msgs

    def apply(self, lus, k):
        """Apply received decrements one at a time (any order gives the same result)."""
        pushed, lmin = 0, None
        for lu in lus:
            old = self.deg[lu]
            self.deg[lu] = old - 1
            if old == k + 1:
                self.deg[lu] += REMOVED
                self.next_inbox.append(lu)
                pushed += 1
            elif k + 1 < old < DEAD:
                lmin = old - 1 if lmin is None else min(lmin, old - 1)
        return pushed, lmin

    def swap(self):
        self.inbox, self.next_inbox = self.next_inbox, []


def _min(a, b):
    return b if a is None else (a if b is None else min(a, b))


def run_rank(rank: Rank, n, exchange, allreduce_sum, allreduce_min):
    """The protocol of one rank.  exchange(msgs: {owner: list}) -> list of
    local ids addressed to this rank; allreduce_sum / allreduce_min over ranks
    (allreduce_min ignores None)."""
    iso, m0 = rank.init_stats()
    removed = allreduce_sum(iso)
    lmin = allreduce_min(m0)
    k = -1
    levels = 1 if removed else 0
    while removed < n:
        k = max(k + 1, lmin)
        pushed, smin = rank.scan(k)
        lvl_min = smin
        pushed = allreduce_sum(pushed)
        lvl_removed = pushed
        while pushed:
            msgs = rank.walk(k)
            got = exchange(msgs)
            p, m = rank.apply(got, k)
            lvl_min = _min(lvl_min, m)
            rank.swap()
            pushed = allreduce_sum(p)
            lvl_removed += pushed
        removed += lvl_removed
        if lvl_removed:
            levels += 1
        lmin = allreduce_min(lvl_min)
    return rank.core, levels


def run_in_process(rowptr, colidx, P):
    """P ranks in this process (lock-step: every rank's phase, then the exchange)."""
    rowptr = np.asarray(rowptr, dtype=np.int64)
    colidx = np.asarray(colidx, dtype=np.int64)
    n = rowptr.size - 1
    ranges = [((n * r) // P, (n * (r + 1)) // P) for r in range(P)]
    ranks = []
    for vb, ve in ranges:
        a0, a1 = rowptr[vb], rowptr[ve]
        ranks.append(Rank(rowptr[vb:ve + 1] - a0, colidx[a0:a1], vb, ve, ranges))
    if n == 0:
        return np.zeros(0, dtype=np.int64), 0
    removed = sum(r.init_stats()[0] for r in ranks)
    lmin = None
    for r in ranks:
        lmin = _min(lmin, r.init_stats()[1])
    k, levels = -1, (1 if removed else 0)
    while removed < n:
        k = max(k + 1, lmin)
        lvl_min, pushed = None, 0
        for r in ranks:
            p, m = r.scan(k)
            pushed += p
            lvl_min = _min(lvl_min, m)
        lvl_removed = pushed
        while pushed:
            inbox = [[] for _ in range(P)]
            for r in ranks:
                for o, lst in r.walk(k).items():
                    inbox[o].extend(lst)
            pushed = 0
            for o, r in enumerate(ranks):
                p, m = r.apply(inbox[o], k)
                pushed += p
                lvl_min = _min(lvl_min, m)
                r.swap()
            lvl_removed += pushed
        removed += lvl_removed
        levels += 1 if lvl_removed else 0
        lmin = lvl_min
    return np.concatenate([r.core for r in ranks]), levels
