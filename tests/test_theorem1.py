"""Theorem-1 pins of the MIR predicate by schedule enumeration.

Theorem 1: a program is free of data mapping issues if (1) it is
free of data races and (2) the serialized schedule (nowait regions executed
synchronously) shows no issue.  The oracle reports MIR for the races
among mapping-relevant ops (reading Z10: two ops on one word conflict if one
is write-class; a race needs an op of an unjoined nowait task).

Pins:
  * soundness: oracle reports nothing on the serialized trace  =>  every
    legal schedule is clean under Definition 1 (value simulator);
  * every reported MIR has a witness: an op of some nowait task instance on
    the same word, conflicting, whose join comes after the reported record,
    found by a brute-force pair search independent of the oracle's log; and
    conversely every record with a witness is reported (reading Z11: one MIR
    triple at the later op of each racing pair's word).
"""
import numpy as np

from gen.trace import MAP, OP, UPD, encode
from valuesim import schedule_issues

A = 0x4000  # one 8-byte word
HOST_OPS = ["RH", "WH", "RT", "WT", "UPT", "UPH"]   # RT/WT here = synchronous target regions
TASK_OPS = ["RT", "WT", "UPT", "UPH"]


def rec_of(name):
    return {"RH": encode(OP.RH, A, 8), "WH": encode(OP.WH, A, 8),
            "RT": encode(OP.RT, A, 8), "WT": encode(OP.WT, A, 8),
            "UPT": encode(OP.UPDATE, A, 8, arg=UPD.TO),
            "UPH": encode(OP.UPDATE, A, 8, arg=UPD.FROM)}[name]


def random_program(rs, ntasks, read_bias=0.0):
    """Items: ('h', op) host op, ('t', k, [ops]) nowait launch of task k, ('s', k) taskwait.
    With read_bias, ops are reads with that probability (race-free concurrency)."""
    items = []
    launched = []
    for _ in range(rs.integers(2, 6)):
        r = rs.random()
        if r < 0.45 or len(launched) == ntasks and r < 0.8:
            items.append(("h", ("RH", "RT")[rs.integers(2)] if rs.random() < read_bias
                           else HOST_OPS[rs.integers(len(HOST_OPS))]))
        elif len(launched) < ntasks and r < 0.8:
            k = len(launched) + 1
            ops = ["RT" if rs.random() < read_bias else TASK_OPS[rs.integers(len(TASK_OPS))]
                   for _ in range(rs.integers(1, 3))]
            items.append(("t", k, ops))
            launched.append(k)
        else:
            items.append(("s", 0xFFFF if rs.random() < 0.5 or not launched
                          else launched[rs.integers(len(launched))]))
    return items


def serialize(items):
    """Serialized trace (Theorem 1(2)): prologue, items, SYNC all, epilogue."""
    recs = [encode(OP.WH, A, 8), encode(OP.MAP_ENTER, A, 8, arg=MAP.TOFROM)]
    for it in items:
        if it[0] == "h":
            recs.append(rec_of(it[1]))
        elif it[0] == "t":
            recs.append(encode(OP.TASK_BEGIN, task=it[1]))
            recs.extend(rec_of(o) for o in it[2])
            recs.append(encode(OP.TASK_END, task=it[1]))
        else:
            recs.append(encode(OP.SYNC, task=it[1]))
    recs.append(encode(OP.SYNC, task=0xFFFF))
    recs.append(encode(OP.MAP_EXIT, A, 8, arg=MAP.TOFROM))
    recs.append(encode(OP.RH, A, 8))
    return recs


def schedules(items):
    """All legal interleavings, as lists of word-op names (the host continues
    after launching a nowait region; a taskwait waits for it)."""
    host = []          # host word-ops in order, with markers for launches and syncs
    tasks = {}
    for it in items:
        if it[0] == "h":
            host.append(("op", it[1]))
        elif it[0] == "t":
            host.append(("launch", it[1]))
            tasks[it[1]] = it[2]
        else:
            host.append(("sync", it[1]))
    host.append(("sync", 0xFFFF))
    out = []

    def rec(hi, state, acc):
        # state: dict task -> (launched?, next op index)
        # option 1: run next task op of any launched, unfinished task
        for k, (launched, nxt) in state.items():
            if launched and nxt < len(tasks[k]):
                st = dict(state); st[k] = (True, nxt + 1)
                rec(hi, st, acc + [tasks[k][nxt]])
        # option 2: advance the host
        if hi == len(host):
            if all(nxt == len(tasks[k]) for k, (_, nxt) in state.items()):
                out.append(acc)
            return
        kind, v = host[hi]
        if kind == "op":
            rec(hi + 1, state, acc + [v])
        elif kind == "launch":
            st = dict(state); st[v] = (True, 0)
            rec(hi + 1, st, acc)
        else:  # sync: every finished-launch task with matching id must be complete
            for k, (launched, nxt) in state.items():
                if launched and (v == 0xFFFF or v == k) and nxt < len(tasks[k]):
                    return
            rec(hi + 1, state, acc)

    rec(0, {k: (False, 0) for k in tasks}, [])
    return out


def to_word_ops(ops):
    pro = [("WH", 0), ("NEW", 0), ("UPT", 0)]
    epi = [("UPH", 0), ("DEL", 0), ("RH", 0)]
    name = {"RH": "RH", "WH": "WH", "RT": "RT", "WT": "WT", "UPT": "UPT", "UPH": "UPH"}
    return pro + [(name[o], 0) for o in ops] + epi


def witness(recs, idx):
    """Brute-force: some nowait task op on A before idx, conflicting, whose task's
    first matching SYNC after its TASK_END is after idx."""
    ops = []
    cur = 0
    for i, (w0, w1) in enumerate(recs):
        op = (w0 >> 48) & 0xFF
        if op == OP.TASK_BEGIN:
            cur = (w1 >> 48, i)
        elif op == OP.TASK_END:
            cur = 0
        elif op in (OP.RH, OP.WH, OP.RT, OP.WT, OP.UPDATE, OP.MAP_ENTER, OP.MAP_EXIT):
            ops.append((i, cur, op not in (OP.RH, OP.RT)))
    me = [o for o in ops if o[0] == idx]
    if not me:
        return False
    _, my_task, my_w = me[0]
    for i, task, w in ops:
        if i >= idx or task == 0 or task == my_task or not (w or my_w):
            continue
        tid, tb = task
        end = next(j for j in range(tb, len(recs)) if (recs[j][0] >> 48) & 0xFF == OP.TASK_END)
        join = next((j for j in range(end, len(recs)) if (recs[j][0] >> 48) & 0xFF == OP.SYNC
                     and (recs[j][1] >> 48) in (tid, 0xFFFF)), len(recs))
        if join > idx:
            return True
    return False


def _run(orc, ntasks, nprog, seed, read_bias=0.0):
    rs = np.random.default_rng(seed)
    clean = racy = multi = 0
    for _ in range(nprog):
        items = random_program(rs, ntasks, read_bias)
        recs = serialize(items)
        res = orc.replay(np.array(recs, dtype=np.uint64).reshape(-1, 2), A, 8)
        assert res.rc == 0
        t = res.triples()
        if not t:
            clean += 1
            sch = schedules(items)
            multi += len(sch) > 1
            for sched in sch:
                assert not schedule_issues(to_word_ops(sched)), (items, sched)
        for w, i, k in t:
            if k == 3:
                racy += 1
                assert witness(recs, i), (items, i)
        # Z11 attribution, both ways: a record is reported as MIR exactly when the
        # brute-force pair search finds it the later op of a race
        mir_at = {i for _, i, k in t if k == 3}
        for idx in range(len(recs)):
            assert witness(recs, idx) == (idx in mir_at), (items, idx)
        if t and all(k == 3 for _, _, k in t):
            # negative control: a MIR-only program usually has an unclean schedule
            pass
    return clean, racy, multi


def test_theorem1_one_task(orc):
    clean, racy, multi = _run(orc, 1, 4000, 1)
    assert clean > 100 and racy > 100


def test_theorem1_two_tasks(orc):
    clean, racy, multi = _run(orc, 2, 4000, 2)
    assert clean > 50 and racy > 100


def test_theorem1_concurrent_reads(orc):
    """Read-biased programs: many race-free programs with several legal schedules."""
    clean, racy, multi = _run(orc, 2, 6000, 3, read_bias=0.7)
    assert multi > 300 and racy > 100


def test_mir_is_necessary_for_soundness(orc):
    """Without the MIR part the soundness property fails: MIR-only programs exist
    whose other schedules do show Definition-1 issues."""
    rs = np.random.default_rng(4)
    found = 0
    for _ in range(2000):
        items = random_program(rs, 2)
        recs = serialize(items)
        t = orc.replay(np.array(recs, dtype=np.uint64).reshape(-1, 2), A, 8).triples()
        if t and all(k == 3 for _, _, k in t):
            found += any(schedule_issues(to_word_ops(s)) for s in schedules(items))
    assert found > 50


# ---- depend (reading Z22) --------------------------------------------
def random_program_dep(rs, ntasks, read_bias=0.0):
    """As random_program, but a launched task may depend on an earlier one:
    ('t', k, ops, dep) with dep = an earlier task id or 0."""
    items = []
    launched = []
    for it in random_program(rs, ntasks, read_bias):
        if it[0] == "t":
            dep = int(launched[rs.integers(len(launched))]) if launched and rs.random() < 0.7 else 0
            items.append(("t", it[1], it[2], dep))
            launched.append(it[1])
        else:
            items.append(it)
    return items


def serialize_dep(items):
    recs = [encode(OP.WH, A, 8), encode(OP.MAP_ENTER, A, 8, arg=MAP.TOFROM)]
    for it in items:
        if it[0] == "h":
            recs.append(rec_of(it[1]))
        elif it[0] == "t":
            recs.append(encode(OP.TASK_BEGIN, task=it[1]))
            if it[3]:
                recs.append(encode(OP.TASK_DEPEND, task=it[3]))
            recs.extend(rec_of(o) for o in it[2])
            recs.append(encode(OP.TASK_END, task=it[1]))
        else:
            recs.append(encode(OP.SYNC, task=it[1]))
    recs.append(encode(OP.SYNC, task=0xFFFF))
    recs.append(encode(OP.MAP_EXIT, A, 8, arg=MAP.TOFROM))
    recs.append(encode(OP.RH, A, 8))
    return recs


def schedules_dep(items):
    """Legal interleavings: a task runs its ops after launch and after its
    dependency's ops have all run; a taskwait waits for the tasks it names."""
    host, tasks, dep = [], {}, {}
    for it in items:
        if it[0] == "h":
            host.append(("op", it[1]))
        elif it[0] == "t":
            host.append(("launch", it[1]))
            tasks[it[1]] = it[2]
            dep[it[1]] = it[3]
        else:
            host.append(("sync", it[1]))
    host.append(("sync", 0xFFFF))
    out = []

    def done(state, k):
        return state[k][0] and state[k][1] == len(tasks[k])

    def rec(hi, state, acc):
        for k, (launched, nxt) in state.items():
            if launched and nxt < len(tasks[k]) and (not dep[k] or done(state, dep[k])):
                st = dict(state); st[k] = (True, nxt + 1)
                rec(hi, st, acc + [tasks[k][nxt]])
        if hi == len(host):
            if all(nxt == len(tasks[k]) for k, (_, nxt) in state.items()):
                out.append(acc)
            return
        kind, v = host[hi]
        if kind == "op":
            rec(hi + 1, state, acc + [v])
        elif kind == "launch":
            st = dict(state); st[v] = (True, 0)
            rec(hi + 1, st, acc)
        else:
            for k, (launched, nxt) in state.items():
                if launched and (v == 0xFFFF or v == k) and nxt < len(tasks[k]):
                    return
            rec(hi + 1, state, acc)

    rec(0, {k: (False, 0) for k in tasks}, [])
    return out


def witness_dep(recs, idx):
    """Brute force with dependencies: an earlier conflicting op of another task that
    is not an ancestor of the current one and not yet complete at idx (complete =
    a SYNC naming it or one of its dependants after that dependant's end)."""
    ops, dep, ends, cur = [], {}, {}, 0
    for i, (w0, w1) in enumerate(recs):
        op = (w0 >> 48) & 0xFF
        if op == OP.TASK_BEGIN:
            cur = int(w1 >> 48); dep[cur] = 0
        elif op == OP.TASK_DEPEND:
            dep[cur] = int(w1 >> 48)
        elif op == OP.TASK_END:
            ends[cur] = i; cur = 0
        elif op in (OP.RH, OP.WH, OP.RT, OP.WT, OP.UPDATE, OP.MAP_ENTER, OP.MAP_EXIT):
            ops.append((i, cur, op not in (OP.RH, OP.RT)))

    def ancestors(t):
        a = set()
        while dep.get(t):
            t = dep[t]; a.add(t)
        return a

    def complete_at(t):
        js = [len(recs)]
        for u in [t] + [u for u in dep if t in ancestors(u)]:
            for j in range(ends[u], len(recs)):
                if (recs[j][0] >> 48) & 0xFF == OP.SYNC and (recs[j][1] >> 48) in (u, 0xFFFF):
                    js.append(j)
                    break
        return min(js)

    me = [o for o in ops if o[0] == idx]
    if not me:
        return False
    _, my_task, my_w = me[0]
    anc = ancestors(my_task) if my_task else set()
    for i, task, w in ops:
        if i >= idx or task == 0 or task == my_task or task in anc or not (w or my_w):
            continue
        if complete_at(task) > idx:
            return True
    return False


def _run_dep(orc, ntasks, nprog, seed, read_bias=0.0):
    rs = np.random.default_rng(seed)
    clean = racy = removed = 0
    for _ in range(nprog):
        items = random_program_dep(rs, ntasks, read_bias)
        recs = serialize_dep(items)
        res = orc.replay(np.array(recs, dtype=np.uint64).reshape(-1, 2), A, 8)
        assert res.rc == 0
        t = res.triples()
        if not t:
            clean += 1
            for sched in schedules_dep(items):
                assert not schedule_issues(to_word_ops(sched)), (items, sched)
        for w, i, k in t:
            if k == 3:
                racy += 1
                assert witness_dep(recs, i), (items, i)
        # the same program without its depend records reports at least as many races
        plain = [r for r in recs if (r[0] >> 48) & 0xFF != OP.TASK_DEPEND]
        n_plain = sum(k == 3 for _, _, k in
                      orc.replay(np.array(plain, dtype=np.uint64).reshape(-1, 2), A, 8).triples())
        n_dep = sum(k == 3 for _, _, k in t)
        assert n_plain >= n_dep
        removed += n_plain > n_dep
    return clean, racy, removed


def test_theorem1_depend(orc):
    """Z22 pinned by schedule enumeration: oracle-clean => every schedule that
    respects the dependencies is clean; every MIR has a witness outside the
    current task's ancestors; depend only ever removes races, and does."""
    clean, racy, removed = _run_dep(orc, 3, 4000, 5)
    assert clean > 50 and racy > 100 and removed > 100
