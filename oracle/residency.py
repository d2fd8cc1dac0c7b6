"""Context-switch residency oracle.

Paper: the context manager stashes the whole supernet in pinned CPU memory,
prefetches the predicted next tasks (2 tasks) and evicts finished context, and
delays a copy to GPU until evictions free room under a memory limit.  Reading A9:
residency is decided by Belady's rule over the known per-stage plan under a byte budget,
with write-back on eviction only if the candidate was updated since it was loaded.

    U_K[i] = candidates of stage K's blocks used by task i (F and B both use them).
    Before task i: need = U[i] u ... u U[i+L'-1], L' <= L the largest depth that fits.
    If U[i] alone does not fit -> budget error.
    While bytes(resident u need) > budget: evict from resident \\ need the candidate with
    the farthest next use (never = infinity; ties -> lowest uid = b*n + c).
    Load the missing members of need in next-use order (ties -> lowest uid).
"""
INF = float("inf")


class BudgetError(Exception):
    pass


def stage_uses(order_K, choices, blocks_K, n):
    """U_K[i] as sets of uids for stage K's ordered task list [(kind, y)]."""
    return [{b * n + int(choices[y][b]) for b in blocks_K} for _, y in order_K]


def simulate_residency(uses, kinds, nbytes, budget, L=2, horizon=None):
    """uses: list of uid sets per task; kinds: 0/1 per task (B writes => dirty);
    nbytes: {uid: bytes}; budget: bytes (0 = everything resident, no traffic).
    horizon: reading A26 — "next use" only looks at tasks [i, i + horizon) (None = the whole
    plan), so the decision before task i needs only the plan up to i + horizon - 1, which a
    streaming executor knows without waiting for the end of the stream.

    Returns dict(events=[(op, i, uid)], writebacks=[(i, uid)]) with op in {"LOAD", "EVICT"}.
    """
    events, writebacks = [], []
    if budget == 0:
        return dict(events=events, writebacks=writebacks)
    T = len(uses)
    resident, dirty = set(), set()

    def next_use(uid, i):
        end = T if horizon is None else min(T, i + horizon)
        for j in range(i, end):
            if uid in uses[j]:
                return j
        return INF

    size = lambda s: sum(nbytes[u] for u in s)                      # noqa: E731
    for i in range(T):
        if size(uses[i]) > budget:
            raise BudgetError(f"task {i} needs {size(uses[i])} > budget {budget}")
        need = set(uses[i])
        for depth in range(2, L + 1):
            cand = set().union(*uses[i:i + depth])
            if i + depth - 1 < T and size(cand) <= budget:
                need = cand
            else:
                break
        while size(resident | need) > budget:
            victims = sorted(resident - need, key=lambda u: (-next_use(u, i), u))
            v = victims[0]
            resident.discard(v)
            events.append(("EVICT", i, v))
            if v in dirty:
                writebacks.append((i, v))
                dirty.discard(v)
        for u in sorted(need - resident, key=lambda u: (next_use(u, i), u)):
            resident.add(u)
            events.append(("LOAD", i, u))
        if kinds[i] == 1:
            dirty |= uses[i]
    return dict(events=events, writebacks=writebacks)
