"""CSP scheduling oracle (plus the balanced partition).

Definitions followed:
* Def.2 dependency preservation: if SN_x and SN_y (x < y) choose the same layer l,
  SN_y's READ and WRITE of l wait for SN_x's WRITE of l.
* Alg.2: a queued forward ``qval`` on stage K is blocked if any earlier
  ``wval`` not in L_f has one of qval's stage-K layers.
* Alg.1 + P:L154/P:L225: backward first, lower ID first.

Readings: layer id = globally unique (block, choice) (A1); strict
backward-first with lowest-ID pending backward (A5); queued forwards scanned in ascending ID
(A6); the stage-0 window W over the lowest unfinished ID (A7); logical integer time with
completions/deliveries applied before decisions (A8); fixed contiguous partition (A12).
"""
from itertools import combinations

import numpy as np


# --------------------------------------------------------------------------------------
# O3: dependency table
# --------------------------------------------------------------------------------------
def dep_table(choices):
    """dep[y][b] = the latest x < y with c_x[b] == c_y[b], else -1 (written out as a scan)."""
    N, m = len(choices), len(choices[0])
    dep = np.full((N, m), -1, dtype=np.int64)
    for y in range(N):
        for b in range(m):
            for x in range(y - 1, -1, -1):
                if choices[x][b] == choices[y][b]:
                    dep[y, b] = x
                    break
    return dep


def stage_blocks(stage_of_block, K):
    return [b for b, s in enumerate(stage_of_block) if s == K]


def deps(choices, stage_of_block, y, K):
    """deps(y,K) = {dep[y][b] : b in blocks(K)} minus {-1} (O3)."""
    dep = dep_table(choices[: y + 1])
    return {int(dep[y, b]) for b in stage_blocks(stage_of_block, K)} - {-1}


# --------------------------------------------------------------------------------------
# O5: Algorithm 2, verbatim
# --------------------------------------------------------------------------------------
def literal_alg2(Lq, Lf, L_SN, K, stage_of_block):
    """Algorithm 2 line by line.

    Lq: queue list of subnet ids (scanned in the given order); Lf: finished list;
    L_SN[y]: subnet y as a list of layer ids (b, c); K: stage.  Returns (qidx, qval)."""
    for qidx, qval in enumerate(Lq):                          # line 2
        scheduled = True                                     # line 3
        for wval in range(0, qval):                          # line 4: [0, qval-1]
            if wval in Lf:                                   # line 5
                continue                                     # line 6
            layers_w = set(L_SN[wval])
            for l in L_SN[qval]:                             # line 7: l in L_SN[qval][K]
                if stage_of_block[l[0]] != K:
                    continue
                if l in layers_w:                            # line 8
                    scheduled = False                        # line 9
                    break                                    # line 10
            if not scheduled:
                break
        if scheduled:                                        # line 11
            return qidx, qval                                # line 12
    return -1, -1                                            # line 13


# --------------------------------------------------------------------------------------
# Partition ("D-partition ... roughly the same execution time"; reading A12)
# --------------------------------------------------------------------------------------
def balanced_partition(block_cost, D):
    """Contiguous partition of blocks into D non-empty stages minimising the max stage
    cost; ties -> lexicographically smallest split points.  Brute force over all splits."""
    m = len(block_cost)
    assert 1 <= D <= m
    best, best_splits = None, None
    for splits in combinations(range(1, m), D - 1):          # lexicographic order
        bounds = (0,) + splits + (m,)
        worst = max(sum(block_cost[bounds[i]:bounds[i + 1]]) for i in range(D))
        if best is None or worst < best:
            best, best_splits = worst, bounds
    sob = np.zeros(m, dtype=np.int32)
    for K in range(D):
        sob[best_splits[K]:best_splits[K + 1]] = K
    return sob


def block_partition_cost(cost_f, cost_b):
    """Per-block partition weight: sum over choices of (cf + cb) (n * the mean, A12)."""
    return [int(np.sum(cost_f[b]) + np.sum(cost_b[b])) for b in range(len(cost_f))]


# --------------------------------------------------------------------------------------
# O2: logical-time discrete-event CSP schedule
# --------------------------------------------------------------------------------------
def task_costs(choices, stage_of_block, cost_f, cost_b, D):
    """cf[K][y] = max(1, sum_{b in blocks(K)} cost_f[b][c_y[b]]) (same for cb)."""
    N = len(choices)
    cf = np.zeros((D, N), dtype=np.int64)
    cb = np.zeros((D, N), dtype=np.int64)
    for K in range(D):
        for y in range(N):
            sf = sum(int(cost_f[b][choices[y][b]]) for b in stage_blocks(stage_of_block, K))
            sb = sum(int(cost_b[b][choices[y][b]]) for b in stage_blocks(stage_of_block, K))
            cf[K, y], cb[K, y] = max(1, sf), max(1, sb)
    return cf, cb


def simulate_csp(choices, stage_of_block, D, W, cf, cb, lam=0, policy=0, ignore_deps=False,
                 admit=None, sync="csp", bulk=0, observe=None):
    """O2.  Returns dict(trace=[(t, K, kind, y)], makespan, order=[[(kind, y)] per stage],
    stall=[ticks per stage], bubble=[ticks per stage]).  An idle stage is *stalled* while a
    queued forward is blocked by a dependency and in a *bubble* while nothing is queued
    (dependency stall vs bubble).

    kind: 0 = F (forward), 1 = B (backward).  cf, cb: int [D][N] task costs (>= 1).
    policy 0: strict backward-first (A5).  policy 1: after a backward, try one forward
    first (Alg.1's alternation).  ``ignore_deps`` gives the no-dependency upper bound used
    in the sweep report (not CSP).  ``admit(K, inF_K, fin_K) -> y or None`` replaces the
    dependency-table admission rule (used to cross-check against Algorithm 2 verbatim).

    ``sync`` (include/naspipe.h naspipe_sync) changes only the admission:
    "csp" the method; "serial" NASPipe w/o scheduler as P:L454 words it ("had to finish the
    execution of a pipeline before injecting the next pipeline"): the window forced to
    W = 1, one subnet in flight; "inorder" the in-order-admission variant of the ablation
    (Fig.6): only the lowest-id
    queued forward may start, a blocked head blocks the stage; "asp" (PipeDream-style,
    P:L123) dependencies ignored; "bsp" (GPipe/Retiarii): dependencies ignored inside
    bulks of ``bulk`` consecutive subnets (0 = 4 D), a stage runs any queued forward before
    a backward, and stage 0 admits bulk k only once every subnet of bulk k-1 finished on
    stage 0 (the flush: a subnet's stage-0 backward is its last task).

    ``observe(t, K, kind, y, queued, finished)``, if given, sees every task start with the
    stage's queued forwards and finished set just before it (an observer: no effect)."""
    N = len(choices)
    G = bulk if bulk > 0 else 4 * D
    if sync == "serial":   # "w/o scheduler" as P:L454 words it: one pipeline (subnet) at a time (A32)
        W = 1
    no_deps = ignore_deps or sync in ("asp", "bsp")
    dep_sets = [[set() if no_deps else deps(choices, stage_of_block, y, K)
                 for y in range(N)] for K in range(D)]
    fin = [set() for _ in range(D)]
    inF = [set() for _ in range(D)]
    inB = [set() for _ in range(D)]
    started0 = set()
    busy = [None] * D              # (end_time, kind, y)
    last_kind = [None] * D
    deliveries = []                # (time, kind, K, y): kind 0 -> inF[K], 1 -> inB[K]
    trace, order = [], [[] for _ in range(D)]
    stall, bubble = [0] * D, [0] * D
    t = 0
    done0 = 0
    while True:
        # (1) completions at t, then deliveries with time <= t
        for K in range(D):
            if busy[K] is not None and busy[K][0] == t:
                _, kind, y = busy[K]
                busy[K] = None
                if kind == 0:
                    if K < D - 1:
                        deliveries.append((t + lam, 0, K + 1, y))
                    else:
                        inB[K].add(y)
                else:
                    fin[K].add(y)
                    if K > 0:
                        deliveries.append((t + lam, 1, K - 1, y))
                    else:
                        done0 += 1
        keep = []
        for dv in deliveries:
            if dv[0] <= t:
                (inF if dv[1] == 0 else inB)[dv[2]].add(dv[3])
            else:
                keep.append(dv)
        deliveries = keep
        if done0 == N:
            return dict(trace=trace, makespan=t, order=order, stall=stall, bubble=bubble)
        # (2) stage-0 source under the window
        wm0 = min([y for y in range(N) if y not in fin[0]], default=N)
        hi = (wm0 // G + 1) * G if sync == "bsp" else wm0 + W
        for y in range(N):
            if y < hi and y not in started0:
                inF[0].add(y)
        # (3) decisions on idle stages
        for K in range(D):
            if busy[K] is not None:
                continue
            if admit is not None:
                first = admit(K, set(inF[K]), set(fin[K]))
            elif sync == "inorder":
                head = min(inF[K]) if inF[K] else None
                first = head if head is not None and dep_sets[K][head] <= fin[K] else None
            else:
                admissible = sorted(y for y in inF[K] if dep_sets[K][y] <= fin[K])
                first = admissible[0] if admissible else None
            choose = None
            if sync == "bsp" and first is not None:
                choose = (0, first)
            elif policy == 1 and last_kind[K] == 1 and first is not None:
                choose = (0, first)
            elif inB[K]:
                choose = (1, min(inB[K]))
            elif first is not None:
                choose = (0, first)
            if choose is None:
                continue
            kind, y = choose
            if observe is not None:
                observe(t, K, kind, y, sorted(inF[K]), set(fin[K]))
            if kind == 0:
                inF[K].discard(y)
                if K == 0:
                    started0.add(y)
                busy[K] = (t + int(cf[K][y]), 0, y)
            else:
                inB[K].discard(y)
                busy[K] = (t + int(cb[K][y]), 1, y)
            last_kind[K] = kind
            trace.append((t, K, kind, y))
            order[K].append((kind, y))
        # (4) advance time
        nxt = [b[0] for b in busy if b is not None] + [dv[0] for dv in deliveries]
        assert nxt, "CSP simulation stalled (no pending event)"
        dt = min(nxt) - t
        for K in range(D):
            if busy[K] is None:
                if inF[K]:
                    stall[K] += dt
                else:
                    bubble[K] += dt
        t = min(nxt)


# --------------------------------------------------------------------------------------
# O4: trace checker (precedence + Table 4 access pattern)
# --------------------------------------------------------------------------------------
def check_trace(trace, choices, stage_of_block, D):
    """Returns a list of violations (empty == valid CSP trace).

    trace: [(t, K, kind, y)] task starts in nondecreasing t, or per-stage order lists
    converted by the caller.  Checks: F(y,K) before B(y,K); F(y,K) after F(y,K-1);
    B(y,K) after B(y,K+1); for every candidate l its accesses read F(x1) B(x1) F(x2) B(x2)...
    with x1 < x2 < ... (Table 4)."""
    errs = []
    pos = {}
    for idx, (t, K, kind, y) in enumerate(trace):
        pos[(kind, y, K)] = (t, idx)
    N = len(choices)
    for y in range(N):
        for K in range(D):
            if (0, y, K) not in pos or (1, y, K) not in pos:
                errs.append(f"missing task y={y} K={K}")
                continue
            if pos[(0, y, K)] >= pos[(1, y, K)]:
                errs.append(f"B before F y={y} K={K}")
            if K > 0 and pos[(0, y, K)] <= pos[(0, y, K - 1)]:
                errs.append(f"F({y},{K}) not after F({y},{K-1})")
            if K < D - 1 and pos[(1, y, K)] <= pos[(1, y, K + 1)]:
                errs.append(f"B({y},{K}) not after B({y},{K+1})")
    # per-candidate access sequence in trace order on its owning stage
    acc = {}
    for (t, K, kind, y) in trace:
        for b in stage_blocks(stage_of_block, K):
            acc.setdefault((b, int(choices[y][b])), []).append((kind, y))
    for l, seq in acc.items():
        users = sorted({y for _, y in seq})
        expect = [(k, y) for y in users for k in (0, 1)]
        if seq != expect:
            errs.append(f"candidate {l} access order {seq} != {expect}")
    return errs


def expected_versions(choices):
    """Version invariant: v(y, (b,c)) = #{x < y : c_x[b] == c}."""
    N, m = len(choices), len(choices[0])
    v = np.zeros((N, m), dtype=np.int64)
    for y in range(N):
        for b in range(m):
            v[y, b] = sum(1 for x in range(y) if choices[x][b] == choices[y][b])
    return v


# --------------------------------------------------------------------------------------
# per-subnet balanced partitions with layer mirroring
# --------------------------------------------------------------------------------------
def subnet_partitions(choices, cost_f, cost_b, D):
    """"The partition is a D-partition ... of a subnet's sequential list of layers,
    with each partition having roughly the same execution time": subnet y's stage of block
    b from balanced_partition over y's own per-block costs cf(b, c_y[b]) + cb(b, c_y[b])
    (same tie rule as A12).  Returns int32 [N][m]."""
    return np.array([balanced_partition([int(cost_f[b][c[b]]) + int(cost_b[b][c[b]]) for b in range(len(c))], D)
                     for c in choices], dtype=np.int32)


def simulate_csp_mirrored(choices, sob, D, W, cost_f, cost_b, lam=0, lam_w=0):
    """O2 with a stage assignment per subnet (reading A31).  sob[y][b] = stage of block b in
    subnet y; a candidate used by subnets on different stages is mirrored.

    Task costs: cf[K][y] = max(1, sum of cost_f[b][c_y[b]] over y's blocks on K) (cb alike).
    Dependency (Def.2): F(y, K) may start at t only if, for every block b of y on K
    with an earlier user x = dep[y][b] of candidate (b, c_y[b]), x's WRITE of it — the end of
    B(x, sob[x][b]) — happened at or before t, plus lam_w ticks when sob[x][b] != K (the
    updated parameters are pushed to the mirror).  Everything else is O2: strict
    backward-first, lowest id first, the stage-0 window W, deliveries after lam ticks.
    With sob[y] equal for all y and lam_w = 0 this is simulate_csp.
    Returns dict(trace, makespan, order, stall, bubble)."""
    N, m = len(choices), len(choices[0])
    sob = np.asarray(sob)
    dep = dep_table(choices)
    cf = np.zeros((D, N), dtype=np.int64)
    cb = np.zeros((D, N), dtype=np.int64)
    for y in range(N):
        for K in range(D):
            bl = [b for b in range(m) if sob[y][b] == K]
            cf[K, y] = max(1, sum(int(cost_f[b][choices[y][b]]) for b in bl))
            cb[K, y] = max(1, sum(int(cost_b[b][choices[y][b]]) for b in bl))
    bend = {}                      # (x, K) -> end time of B(x, K)
    inF = [set() for _ in range(D)]
    inB = [set() for _ in range(D)]
    fin0 = set()
    started0 = set()
    busy = [None] * D
    deliveries = []
    trace, order = [], [[] for _ in range(D)]
    stall, bubble = [0] * D, [0] * D
    t = 0

    def ready_at(y, K):
        """Earliest time F(y, K)'s dependencies allow (None while some WRITE is pending)."""
        r = 0
        for b in range(m):
            if sob[y][b] != K or dep[y, b] < 0:
                continue
            x = int(dep[y, b])
            Kx = int(sob[x][b])
            if (x, Kx) not in bend or bend[(x, Kx)] > t:
                return None
            r = max(r, bend[(x, Kx)] + (lam_w if Kx != K else 0))
        return r

    while True:
        for K in range(D):
            if busy[K] is not None and busy[K][0] == t:
                _, kind, y = busy[K]
                busy[K] = None
                if kind == 0:
                    if K < D - 1:
                        deliveries.append((t + lam, 0, K + 1, y))
                    else:
                        inB[K].add(y)
                else:
                    if K > 0:
                        deliveries.append((t + lam, 1, K - 1, y))
                    else:
                        fin0.add(y)
        keep = []
        for dv in deliveries:
            if dv[0] <= t:
                (inF if dv[1] == 0 else inB)[dv[2]].add(dv[3])
            else:
                keep.append(dv)
        deliveries = keep
        if len(fin0) == N:
            return dict(trace=trace, makespan=t, order=order, stall=stall, bubble=bubble)
        wm0 = min([y for y in range(N) if y not in fin0], default=N)
        for y in range(N):
            if y < wm0 + W and y not in started0:
                inF[0].add(y)
        wake = []                  # future times at which a mirror push completes
        for K in range(D):
            if busy[K] is not None:
                continue
            choose = None
            if inB[K]:
                choose = (1, min(inB[K]))
            else:
                for y in sorted(inF[K]):
                    r = ready_at(y, K)
                    if r is None:
                        continue
                    if r <= t:
                        choose = (0, y)
                        break
                    wake.append(r)
            if choose is None:
                continue
            kind, y = choose
            if kind == 0:
                inF[K].discard(y)
                if K == 0:
                    started0.add(y)
                busy[K] = (t + int(cf[K][y]), 0, y)
            else:
                inB[K].discard(y)
                busy[K] = (t + int(cb[K][y]), 1, y)
                bend[(y, K)] = t + int(cb[K][y])
            trace.append((t, K, kind, y))
            order[K].append((kind, y))
        nxt = [b[0] for b in busy if b is not None] + [dv[0] for dv in deliveries] + [w for w in wake if w > t]
        assert nxt, "mirrored CSP simulation stalled (no pending event)"
        dt = min(nxt) - t
        for K in range(D):
            if busy[K] is None:
                if inF[K]:
                    stall[K] += dt
                else:
                    bubble[K] += dt
        t = min(nxt)


def check_trace_mirrored(trace, choices, sob, D, cost_b, lam_w=0):
    """Validity of a mirrored trace: every task once; F(y,K) after F(y,K-1), B(y,K) after
    B(y,K+1), F before B on a stage; and for every candidate l, in start-time order, its
    users' accesses read F(x1) B(x1) F(x2) B(x2) ... with x1 < x2 < ... (Table 4 pattern,
    P:L435) where each F(x_{i+1}) starts no earlier than B(x_i)'s end (+ lam_w across
    stages).  Returns a list of violations."""
    errs = []
    N, m = len(choices), len(choices[0])
    sob = np.asarray(sob)
    pos = {}
    for idx, (t, K, kind, y) in enumerate(trace):
        if (kind, y, K) in pos:
            errs.append(f"task twice {(kind, y, K)}")
        pos[(kind, y, K)] = (t, idx)
    for y in range(N):
        for K in range(D):
            if (0, y, K) not in pos or (1, y, K) not in pos:
                errs.append(f"missing task y={y} K={K}")
                continue
            if pos[(0, y, K)] >= pos[(1, y, K)]:
                errs.append(f"B before F y={y} K={K}")
            if K > 0 and pos[(0, y, K)] <= pos[(0, y, K - 1)]:
                errs.append(f"F({y},{K}) not after F({y},{K-1})")
            if K < D - 1 and pos[(1, y, K)] <= pos[(1, y, K + 1)]:
                errs.append(f"B({y},{K}) not after B({y},{K+1})")
    acc = {}
    for (t, K, kind, y) in trace:
        for b in range(m):
            if sob[y][b] == K:
                acc.setdefault((b, int(choices[y][b])), []).append((t, kind, y, K))
    for l, seq in acc.items():
        users = sorted({y for _, _, y, _ in seq})
        if [(k, y) for _, k, y, _ in seq] != [(k, y) for y in users for k in (0, 1)]:
            errs.append(f"candidate {l} access order {[(k, y) for _, k, y, _ in seq]}")
            continue
        for i in range(1, len(users)):
            tb, Kb = next((t, K) for t, k, y, K in seq if k == 1 and y == users[i - 1])
            cbx = sum(int(cost_b[b][choices[users[i - 1]][b]]) for b in range(m) if sob[users[i - 1]][b] == Kb)
            tf, Kf = next((t, K) for t, k, y, K in seq if k == 0 and y == users[i])
            if tf < tb + max(1, cbx) + (lam_w if Kf != Kb else 0):
                errs.append(f"candidate {l}: F({users[i]}) at {tf} before the WRITE of {users[i - 1]} landed")
    return errs




# --------------------------------------------------------------------------------------
# the Alg.3 context predictor, evaluated against the exact plan
# --------------------------------------------------------------------------------------
def alg3_backward_predictions(choices, stage_of_block, D, W, cf, cb, lam=0):
    """Alg.3's backward branch (its lines 4-8): before B(x, K) runs, the stage
    pre-adds x to a copy of its finished list L_f (reading A10: L' is a copy) and re-runs
    SCHEDULE (Alg.2, literal_alg2) on its queue L_q to predict the forward it will run next,
    whose context it prefetches.  Every B(x, K) start of the O2 plan is replayed with the
    plan's own L_q / L_f at that tick; the prediction is compared with the forward the plan
    actually starts next on K (None if a backward comes first or nothing follows).  The exact
    plan lookahead the executor uses (readings A9, A26) is right by construction.

    Returns [(t, K, x, predicted, actual)] in start order."""
    m = len(choices[0])
    L_SN = [[(b, int(choices[y][b])) for b in range(m)] for y in range(len(choices))]
    starts = []

    def observe(t, K, kind, y, queued, finished):
        starts.append((t, K, kind, y, queued, finished))

    simulate_csp(choices, stage_of_block, D, W, cf, cb, lam=lam, observe=observe)
    out = []
    for i, (t, K, kind, y, queued, finished) in enumerate(starts):
        if kind != 1:
            continue
        _, pred = literal_alg2(queued, sorted(finished | {y}), L_SN, K, stage_of_block)
        nxt = next(((k2, y2) for (_, K2, k2, y2, _, _) in starts[i + 1:] if K2 == K), None)
        actual = nxt[1] if nxt is not None and nxt[0] == 0 else None
        out.append((t, K, y, None if pred < 0 else pred, actual))
    return out
