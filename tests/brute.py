"""Brute-force happens-before race checking for tiny traces — an independent pin for the oracle.

HB is computed by explicit-graph transitive closure, with no vector clocks (SURVEY.md §8(c) "Pins",
VC computation row):
  * program-order edges between consecutive events of the same fiber; a FORK(src→dst) is an event of
    src's program order only, plus one edge from the FORK to dst's next event;
  * for ACQUIRE j on key k: an edge from the last RELEASE_STORE on k before j, and from every RELEASE
    on k after that store (all RELEASEs on k before j if there is no store).
Race sets are derived from the plain definitions (conflicting accesses, at least
one write, no happens-before):
  * all_pairs  — every conflicting unordered pair (a, b, g)
  * per_fiber  — SURVEY.md §8(c) step 3 (last write, last read per fiber since it), filtered by graph HB
"""
from __future__ import annotations

EV_ACCESS, EV_RELEASE, EV_RELEASE_STORE, EV_ACQUIRE, EV_FORK = 0, 1, 2, 3, 4


def program_fiber(e) -> int:
    """Fiber whose program order contains event e (FORK belongs to its source)."""
    return int(e["a"]) if int(e["kind"]) == EV_FORK else int(e["fiber"])


def hb_closure(events) -> list[int]:
    """reach[i] = bitset of events j > i with i →hb j (strict)."""
    n = len(events)
    succ = [set() for _ in range(n)]
    last_on = {}
    pending_fork: dict[int, list[int]] = {}
    for i in range(n):
        e = events[i]
        f = program_fiber(e)
        if f in last_on:
            succ[last_on[f]].add(i)
        last_on[f] = i
        for src in pending_fork.pop(f, []):
            succ[src].add(i)
        if int(e["kind"]) == EV_FORK:
            pending_fork.setdefault(int(e["fiber"]), []).append(i)
        if int(e["kind"]) == EV_ACQUIRE:
            key = int(e["a"])
            rel = []
            for j in range(i):
                ej = events[j]
                if int(ej["a"]) != key:
                    continue
                if int(ej["kind"]) == EV_RELEASE_STORE:
                    rel = [j]
                elif int(ej["kind"]) == EV_RELEASE:
                    rel.append(j)
            for j in rel:
                succ[j].add(i)
    reach = [0] * n
    for i in range(n - 1, -1, -1):
        r = 0
        for j in succ[i]:
            r |= (1 << j) | reach[j]
        reach[i] = r
    return reach


def granules(e):
    a, n = int(e["a"]), int(e["b"])
    if n == 0:
        return range(0)
    return range(a >> 3, (a + n + 7) >> 3)


def accesses_by_granule(events):
    by = {}
    for i in range(len(events)):
        e = events[i]
        if int(e["kind"]) != EV_ACCESS:
            continue
        for g in granules(e):
            by.setdefault(g, []).append(i)
    return by


def per_fiber_race_set(events, reach=None) -> set[tuple[int, int, int]]:
    reach = hb_closure(events) if reach is None else reach

    def hb(a, b):
        return (reach[a] >> b) & 1

    out = set()
    for g, accs in accesses_by_granule(events).items():
        for jj, b in enumerate(accs):
            fb = int(events[b]["fiber"])
            wb = int(events[b]["mode"]) == 1
            lw = None
            for a in accs[:jj]:
                if int(events[a]["mode"]) == 1:
                    lw = a
            if lw is not None and int(events[lw]["fiber"]) != fb and not hb(lw, b):
                out.add((g, lw, b))
            if wb:
                start = accs.index(lw) + 1 if lw is not None else 0
                last_read = {}
                for a in accs[start:jj]:
                    if int(events[a]["mode"]) == 0:
                        last_read[int(events[a]["fiber"])] = a
                for t, a in last_read.items():
                    if t != fb and not hb(a, b):
                        out.add((g, a, b))
    return out


def all_pairs_race_set(events, reach=None) -> set[tuple[int, int, int]]:
    reach = hb_closure(events) if reach is None else reach
    out = set()
    for g, accs in accesses_by_granule(events).items():
        for x, a in enumerate(accs):
            for b in accs[x + 1:]:
                if int(events[a]["mode"]) == 0 and int(events[b]["mode"]) == 0:
                    continue
                if int(events[a]["fiber"]) == int(events[b]["fiber"]):
                    continue
                if not (reach[a] >> b) & 1:
                    out.add((g, a, b))
    return out


def runs_to_triples(runs) -> set[tuple[int, int, int]]:
    out = set()
    for r in runs:
        for g in range(int(r["g_begin"]), int(r["g_end"])):
            out.add((g, int(r["earlier"]), int(r["later"])))
    return out


def runs_to_triples_in(runs, granules: set) -> set[tuple[int, int, int]]:
    """Triples of `runs` restricted to the given granules (runs may span billions of granules)."""
    import bisect
    gs = sorted(granules)
    out = set()
    for r in runs:
        lo = bisect.bisect_left(gs, int(r["g_begin"]))
        hi = bisect.bisect_left(gs, int(r["g_end"]))
        for g in gs[lo:hi]:
            out.add((g, int(r["earlier"]), int(r["later"])))
    return out


class HBGraph:
    """The same happens-before graph as ``hb_closure`` for traces of any length, queried pair by
    pair (forward search) instead of closed.  The acquire edges of a key are routed through a chain
    of per-key nodes: RELEASE i links into the key's chain at its position, the chain runs forward in
    trace order, a RELEASE_STORE starts a new chain, and ACQUIRE j links from the chain's last node —
    so RELEASE i reaches ACQUIRE j through the chain iff i < j with no RELEASE_STORE on the key in
    between (other than i itself being that store), exactly the edge set of ``hb_closure``."""

    def __init__(self, events):
        n = len(events)
        kind = [int(k) for k in events["kind"]]
        fib = [int(f) for f in events["fiber"]]
        key = [int(a) for a in events["a"]]
        self.n = n
        self.succ: list[list[int]] = [[] for _ in range(n)]
        self.t: list[int] = list(range(n))            # node time (trace position; chain nodes: creation)
        last_on: dict[int, int] = {}
        pending_fork: dict[int, list[int]] = {}
        chain: dict[int, int] = {}                    # key -> last chain node
        for i in range(n):
            k = kind[i]
            f = key[i] if k == EV_FORK else fib[i]
            if f in last_on:
                self.succ[last_on[f]].append(i)
            last_on[f] = i
            for src in pending_fork.pop(f, []):
                self.succ[src].append(i)
            if k == EV_FORK:
                pending_fork.setdefault(fib[i], []).append(i)
            elif k in (EV_RELEASE, EV_RELEASE_STORE):
                node = len(self.succ)
                self.succ.append([])
                self.t.append(i)
                if k == EV_RELEASE and key[i] in chain:
                    self.succ[chain[key[i]]].append(node)
                self.succ[i].append(node)
                chain[key[i]] = node
            elif k == EV_ACQUIRE and key[i] in chain:
                self.succ[chain[key[i]]].append(i)

    def hb(self, a: int, b: int) -> bool:
        """a →hb b (a < b): b reachable from a over edges that never pass b's trace position."""
        seen = {a}
        stack = [a]
        while stack:
            x = stack.pop()
            for y in self.succ[x]:
                if y == b:
                    return True
                if y not in seen and self.t[y] < b:
                    seen.add(y)
                    stack.append(y)
        return False
