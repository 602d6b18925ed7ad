"""Happens-before model of the per-generation halo-exchange schedules of the
multi-process (NCCL) mode — api.cpp iterate_once (serial), iterate_concurrent
(MAPSM_OPT_EXCHANGE_SMS > 0) and iterate_concurrent_ce (MAPSM_EXCHANGE_CE),
DESIGN.md §8 — checked for every rank of a WRAP ring (P = 1: the one-rank
NCCL ring, P = 2: up == down, P = 3) over several generations:

* no data race: any two accesses of the same (rank, buffer, row), at least
  one a write, are ordered by the schedule's stream order, events, NCCL
  matching and copy-engine / mailbox waits;
* every read sees the right generation: the last write before it (in that
  order) produced exactly the generation the Life / conv step needs
  (the two-line boundary exchange of P:L461 §5.1 delivers generation t's
  halo before generation t+1's boundary rows read it).

The model is the schedule as documented in the code (which operations each
launch reads and writes, what each stream waits on); a change of the
schedule there must be mirrored here.  Pure host logic, no GPU."""
import itertools

import pytest


class Sched:
    def __init__(self):
        self.edges = {}
        self.acc = []  # (node, rank, buf, row, is_write, gen_value)
        self.n = 0
        self.names = {}

    def node(self, name):
        k = self.n
        self.n += 1
        self.names[k] = name
        self.edges[k] = set()
        return k

    def edge(self, a, b):
        if a is not None and b is not None:
            self.edges[a].add(b)

    def access(self, node, rank, buf, rows, write, gen):
        for y in rows:
            self.acc.append((node, rank, buf, y, write, gen))

    def closure(self):
        reach = {}
        order = list(range(self.n))  # nodes are created in a topological order
        for v in reversed(order):
            s = set()
            for w in self.edges[v]:
                s.add(w)
                s |= reach[w]
            reach[v] = s
        return reach


def build(P, R, r, gens, mode):
    """The NCCL schedules; mode 'serial' (MAPSM_OPT_EXCHANGE_SMS = 0) or
    'concurrent' (> 0).  Nodes are created in a topological order."""
    S = Sched()
    up = lambda i: (i - 1) % P
    down = lambda i: (i + 1) % P
    top_rows, bot_rows = range(0, r), range(R - r, R)
    bind = S.node("bind")
    for i in range(P):
        S.access(bind, i, 0, range(-r, R + r), True, 0)  # generation 0 with its halos (bind's exchange)
    main = {i: bind for i in range(P)}
    side = {i: bind for i in range(P)}
    ev_b = {i: bind for i in range(P)}
    ev_i = {i: bind for i in range(P)}
    for t in range(gens):
        bi, bo = t % 2, (t + 1) % 2
        B = {i: S.node(f"B{i}({t})") for i in range(P)}
        for i in range(P):
            if mode == "serial":
                S.edge(main[i], B[i])  # main: B(t) after the previous generation's join
            else:
                S.edge(side[i], B[i])  # side: B(t) after X(t-1) ...
                S.edge(ev_i[i], B[i])  # ... and after I(t-1) (wait ev_i)
            S.access(B[i], i, bi, list(range(-r, 2 * r)) + list(range(R - 2 * r, R + r)), False, t)
            S.access(B[i], i, bo, list(top_rows) + list(bot_rows), True, t + 1)
        post = {}
        for i in range(P):  # side: (wait ev_b =) after B(t), the NCCL group is posted
            post[i] = S.node(f"post{i}({t})")
            S.edge(B[i], post[i])
            S.edge(side[i], post[i])
        Ts = []
        for i in range(P):  # my top rows -> up's bottom halo, my bottom rows -> down's top halo
            for dst, rows, halo in ((up(i), top_rows, range(R, R + r)), (down(i), bot_rows, range(-r, 0))):
                T = S.node(f"T{i}->{dst}({t})")
                S.edge(post[i], T)
                S.edge(post[dst], T)  # a transfer needs both sides posted
                S.access(T, i, bo, rows, False, t + 1)
                S.access(T, dst, bo, halo, True, t + 1)
                Ts.append((i, dst, T))
        done = {i: S.node(f"done{i}({t})") for i in range(P)}
        for i, dst, T in Ts:  # a group completes when all its sends and receives did
            S.edge(T, done[i])
            S.edge(T, done[dst])
        I = {i: S.node(f"I{i}({t})") for i in range(P)}
        for i in range(P):
            if mode == "serial":
                S.edge(B[i], I[i])  # main: I(t) after B(t)
            else:
                S.edge(main[i], I[i])  # main: I(t) after I(t-1) ...
                S.edge(ev_b[i], I[i])  # ... and after B(t-1) (wait ev_b)
            S.access(I[i], i, bi, range(0, R), False, t)
            S.access(I[i], i, bo, range(r, R - r), True, t + 1)
        for i in range(P):
            side[i] = done[i]
            if mode == "serial":  # main waits the exchange (ev_h) before the next generation
                j = S.node(f"join{i}({t})")
                S.edge(I[i], j)
                S.edge(done[i], j)
                main[i] = j
            else:
                main[i] = I[i]
                ev_b[i] = B[i]
                ev_i[i] = I[i]
    return S


def build_ce(P, R, r, gens):
    """The copy-engine schedule with the count waits wired generation by generation."""
    S = Sched()
    up = lambda i: (i - 1) % P
    down = lambda i: (i + 1) % P
    top_rows, bot_rows = range(0, r), range(R - r, R)
    bind = S.node("bind")
    for i in range(P):
        S.access(bind, i, 0, range(-r, R + r), True, 0)
    side = {i: bind for i in range(P)}
    main = {i: bind for i in range(P)}
    ev_b = {i: bind for i in range(P)}
    ev_i = {i: bind for i in range(P)}
    counts_prev = {i: [] for i in range(P)}  # count nodes B_i(t) waits for
    for t in range(gens):
        bi, bo = t % 2, (t + 1) % 2
        B = {i: S.node(f"B{i}({t})") for i in range(P)}
        I = {i: S.node(f"I{i}({t})") for i in range(P)}
        counts_next = {i: [] for i in range(P)}
        for i in range(P):
            S.edge(side[i], B[i])
            S.edge(ev_i[i], B[i])
            for c in counts_prev[i]:
                S.edge(c, B[i])
            S.edge(main[i], I[i])
            S.edge(ev_b[i], I[i])
            S.access(B[i], i, bi, list(range(-r, 2 * r)) + list(range(R - 2 * r, R + r)), False, t)
            S.access(B[i], i, bo, list(top_rows) + list(bot_rows), True, t + 1)
            S.access(I[i], i, bi, range(0, R), False, t)
            S.access(I[i], i, bo, range(r, R - r), True, t + 1)
        for i in range(P):
            prev = B[i]
            for dst, rows, halo in ((up(i), top_rows, range(R, R + r)), (down(i), bot_rows, range(-r, 0))):
                D = S.node(f"D{i}->{dst}({t})")
                S.edge(prev, D)
                S.access(D, i, bo, rows, False, t + 1)
                S.access(D, dst, bo, halo, True, t + 1)
                prev = D
            cnt = S.node(f"count{i}({t})")
            S.edge(prev, cnt)
            for dst in {up(i), down(i)}:
                counts_next[dst].append(cnt)
            side[i] = cnt
            main[i] = I[i]
            ev_b[i] = B[i]
            ev_i[i] = I[i]
        counts_prev = counts_next
    return S


def check(S):
    reach = S.closure()
    by_loc = {}
    for a in S.acc:
        by_loc.setdefault(a[1:4], []).append(a)
    for loc, accs in by_loc.items():
        for (n1, *_, w1, g1), (n2, *_, w2, g2) in itertools.combinations(accs, 2):
            if n1 == n2 or not (w1 or w2):
                continue
            assert n2 in reach[n1] or n1 in reach[n2], \
                f"race on rank/buf/row {loc}: {S.names[n1]} vs {S.names[n2]}"
        # every read sees the generation it needs: the HB-latest write before it
        writes = [a for a in accs if a[4]]
        for n, *_, w, g in accs:
            if w:
                continue
            before = [x for x in writes if n in reach[x[0]]]
            assert before, f"{S.names[n]} reads {loc} before any write"
            latest = [x for x in before if not any(y[0] in reach[x[0]] for y in before if y is not x)]
            assert len(latest) == 1 and latest[0][5] == g, \
                f"{S.names[n]} reads {loc}: wants generation {g}, sees {[(S.names[x[0]], x[5]) for x in latest]}"


@pytest.mark.parametrize("P", [1, 2, 3])
@pytest.mark.parametrize("r", [1, 2])
@pytest.mark.parametrize("mode", ["serial", "concurrent"])
def test_nccl_schedules_race_free_and_correct(P, r, mode):
    check(build(P, 4 * r + 2, r, 5, mode))


@pytest.mark.parametrize("P", [1, 2, 3, 4])
@pytest.mark.parametrize("r", [1, 2])
def test_copy_engine_schedule_race_free_and_correct(P, r):
    check(build_ce(P, 4 * r + 2, r, 5))


def test_model_catches_a_missing_wait():
    """Drop the interior's wait on the previous boundary launch: the checker must fail."""
    S = build(2, 6, 1, 4, "concurrent")
    for v in S.edges:
        if S.names[v].startswith("B0("):
            S.edges[v] = {w for w in S.edges[v] if not S.names[w].startswith("I0(")}
    with pytest.raises(AssertionError):
        check(S)


def test_model_catches_a_missing_count_wait():
    """Copy engine: a boundary launch that does not wait for the neighbours' counts races."""
    S = build_ce(2, 6, 1, 4)
    for v in S.edges:
        if S.names[v].startswith("count"):
            S.edges[v] = {w for w in S.edges[v] if not S.names[w].startswith("B")}
    with pytest.raises(AssertionError):
        check(S)
