"""Host-side checks of the dataflow kernels' task queues (apsp_debug_queue: the decoder the
kernels run, evaluated on the host; no GPU): every task of the blocked FW (PAPER.md:62 steps
1-3, Alg. 1 l.3/7/11/17) appears exactly once, on the rank that owns its tile row, and the
queues cannot deadlock — a simulation that runs every rank's queue strictly in order with ONE
worker per rank (the most constrained schedule) completes, with dependencies exactly those
the kernels wait for (per-tile versions, diagonal / panel readiness, panel-parity reuse).
This covers configurations the single test GPU cannot run (P real GPUs)."""
import itertools

import numpy as np
import pytest

P1, P2R, P2C, P3, P3P1, PAIR = 0, 1, 2, 3, 4, 5


def expected_tasks(nb):
    for k in range(nb):
        yield (P1, k, k, k)
        for j in range(nb):
            if j != k:
                yield (P2R, k, k, j)
                yield (P2C, k, j, k)
        for i, j in itertools.product(range(nb), range(nb)):
            if i != k and j != k:
                yield (P3, k, i, j)


def simulate(nb, queues, par=2):
    """queues[r]: array (total, 4) of rank r (P = len(queues); P = 1 single GPU). One worker
    per rank, strictly in queue order; returns True iff every queue drains. par: panel-copy
    parities (2; 4 for the pair schedule, whose round k reuses round k-4's copies)."""
    P = len(queues)
    nl = nb // P
    owner = lambda row: row // nl  # noqa: E731
    ver = np.zeros((nb, nb), dtype=np.int64)  # rounds applied per tile
    p1_done = set()
    p2r_done = set()
    p2c_done = set()
    done2 = np.zeros((P, nb), dtype=np.int64)
    done3 = np.zeros((P, nb), dtype=np.int64)

    def cnt2(r, k):
        l0 = owner(k) == r
        return l0 * (nb - 1) + (nl - l0)

    def cnt3(r, k):
        return (nl - (owner(k) == r)) * (nb - 1)

    parts_done = {}

    def ready(r, t):
        typ, k, i, j = (int(x) for x in t)
        if typ >= 1 << PART_SHIFT:  # a part waits for what its whole task waits for
            return ready(r, (typ & 15, k, i, j))
        if typ == P3P1:  # fused P3(k; k+1,k+1) + P1(k+1) (small-n kernel)
            return (ready(r, (P3, k, i, j)) and
                    (k + 1 < par or all(done2[x, k + 1 - par] >= cnt2(x, k + 1 - par) for x in range(P))))
        if ver[i, j] < k:
            return False
        if typ == PAIR:  # rounds k and k+1 on one tile (pair schedule)
            return all((kk, j) in p2r_done and (kk, i) in p2c_done for kk in (k, k + 1))
        if typ == P3:
            return (k, j) in p2r_done and (k, i) in p2c_done
        if typ == P2C:
            return k in p1_done and (k < par or done3[r, k - par] >= cnt3(r, k - par))
        if typ == P2R:
            return k in p1_done and (k < par or all(done3[x, k - par] >= cnt3(x, k - par) for x in range(P)))
        return k < par or all(done2[x, k - par] >= cnt2(x, k - par) for x in range(P))

    parts_of = {}
    for qu in queues:
        for typ, k, i, j in qu.tolist():
            if typ >= 1 << PART_SHIFT:
                key = (typ & 15, k, i, j)
                parts_of[key] = parts_of.get(key, 0) + 1
    pos = [0] * P
    total = sum(len(q) for q in queues)
    ndone = 0
    while ndone < total:
        progressed = False
        for r in range(P):
            while pos[r] < len(queues[r]) and ready(r, queues[r][pos[r]]):
                typ, k, i, j = (int(x) for x in queues[r][pos[r]])
                if typ >= 1 << PART_SHIFT:  # the whole task's effects once its last part is done
                    key = (typ & 15, k, i, j)
                    parts_done[key] = parts_done.get(key, 0) + 1
                    if parts_done[key] < parts_of[key]:
                        pos[r] += 1
                        ndone += 1
                        progressed = True
                        continue
                    typ = typ & 15
                ver[i, j] = k + 1
                if typ == P3P1:
                    ver[i, j] = k + 2
                    p1_done.add(k + 1)
                    done3[r, k] += 1
                elif typ == PAIR:
                    ver[i, j] = k + 2
                    done3[r, k] += 1
                    done3[r, k + 1] += 1
                elif typ == P1:
                    p1_done.add(k)
                elif typ == P2R:
                    p2r_done.add((k, j))
                    done2[r, k] += 1
                elif typ == P2C:
                    p2c_done.add((k, i))
                    done2[r, k] += 1
                else:
                    done3[r, k] += 1
                pos[r] += 1
                ndone += 1
                progressed = True
        if not progressed:
            return False
    return True


# nb >= 67 takes phase 3's multi-band branch (64-column bands, apsp_df_common.cuh); nb = 130 is a ragged two-band + remainder case
@pytest.mark.parametrize("nb,delay", [(1, 8), (2, 8), (3, 1), (5, 3), (9, 1184), (16, 40), (40, 1), (70, 1184),
                                      (130, 592)])
def test_single_gpu_queue_complete_and_deadlock_free(lib, nb, delay):
    q = lib.apsp_debug_queue(nb, 0, 0, delay)
    assert len(q) == nb ** 3
    assert sorted(map(tuple, q.tolist())) == sorted(expected_tasks(nb))
    assert simulate(nb, [q])


@pytest.mark.parametrize("nb,P,delay", [(1, 1, 8), (2, 2, 8), (3, 3, 1), (4, 2, 5), (8, 4, 2), (8, 8, 1),
                                        (12, 3, 37), (16, 8, 4), (24, 4, 1000), (32, 8, 64), (70, 2, 1184),
                                        (128, 8, 1184), (130, 2, 64)])
def test_sharded_queues_complete_and_deadlock_free(lib, nb, P, delay):
    nl = nb // P
    queues = [lib.apsp_debug_queue(nb, P, q, delay) for q in range(P)]
    allt = []
    for r, qu in enumerate(queues):
        for typ, k, i, j in qu.tolist():
            assert i // nl == r, "task on a row the rank does not own"  # P1 / P2R rows = k, owned
            allt.append((typ, k, i, j))
    assert sorted(allt) == sorted(expected_tasks(nb))
    assert simulate(nb, queues)


def test_sharded_queue_with_one_rank_matches_single_gpu_tasks(lib):
    nb = 10
    a = lib.apsp_debug_queue(nb, 1, 0, 5)
    b = lib.apsp_debug_queue(nb, 0, 0, 5)
    assert sorted(map(tuple, a.tolist())) == sorted(map(tuple, b.tolist()))


def test_simulator_detects_a_deadlocking_order(lib):
    """Pin of the checker itself: swapping a round's phase-1 task behind that round's
    phase-3 tasks cannot complete."""
    nb = 4
    q = lib.apsp_debug_queue(nb, 0, 0, 8).tolist()
    k1 = next(x for x, t in enumerate(q) if t[0] == P1 and t[1] == 1)
    moved = q.pop(k1)
    q.append(moved)
    assert not simulate(nb, [np.array(q)])


def test_bad_arguments(lib):
    with pytest.raises(ValueError):
        lib.apsp_debug_queue(10, 3, 0, 1)  # nb % P != 0
    with pytest.raises(ValueError):
        lib.apsp_debug_queue(8, 4, 4, 1)   # q >= P


PART_SHIFT = 4  # small-n kernel: a part of a split chain panel tile has type base + 16 * (part + 1)


def expand_fused(q):
    parts = {}
    for typ, k, i, j in q.tolist():
        if typ >= 1 << PART_SHIFT:  # one part of a split task: the whole task once its parts are all there
            key = (typ & 15, k, i, j)
            parts.setdefault(key, set()).add((typ >> PART_SHIFT) - 1)
            continue
        if typ == P3P1:
            yield (P3, k, i, j)
            yield (P1, k + 1, i, j)
        elif typ == PAIR:
            yield (P3, k, i, j)
            yield (P3, k + 1, i, j)
        else:
            yield (typ, k, i, j)
    for key, got in parts.items():
        assert got == set(range(len(got))) and len(got) in (2, 4, 8, 16), (key, got)
        yield key


@pytest.mark.parametrize("nb,delay", [(1, 0), (2, 0), (3, 0), (4, 2), (5, 0), (8, 7), (16, 0), (16, 40), (23, 5),
                                      (32, 0), (32, 1000)])
def test_small_kernel_queue_complete_and_deadlock_free(lib, nb, delay):
    """The 64-tile small-n kernel's host-built queue (apsp_fw_small.cu: the 128-tile kernel's segment
    order with F(k) = P3(k; k+1,k+1) fused with P1(k+1)): every blocked-FW task once, and an
    in-order drain with the kernel's exact waits (a fused entry waits for both halves' dependencies)."""
    q = lib.apsp_debug_queue(nb, -1, 0, delay)
    assert sorted(expand_fused(q)) == sorted(expected_tasks(nb))
    S = 16 if nb <= 16 else 8 if nb <= 24 else 4  # default parts per chain panel tile (small_split_for)
    assert len(q) == nb ** 3 - (nb - 1) + 2 * (S - 1) * (nb - 1)
    split = [tuple(t) for t in q.tolist() if t[0] >= 1 << PART_SHIFT]
    assert sorted(split) == sorted((b + ((p + 1) << PART_SHIFT), k, i, j) for k in range(nb - 1) for p in range(S)
                                   for b, i, j in ((P2R, k, k + 1), (P2C, k + 1, k)))
    assert simulate(nb, [q])
    if nb >= 2 and delay == 0:  # round 0's panel tiles right after P1(0), then F(0) (the next diagonal tile) first
        n0 = 2 * (nb - 1) + 2 * (S - 1)
        assert sorted(expand_fused(q[1:1 + n0])) == sorted(
            t for t in expected_tasks(nb) if t[1] == 0 and t[0] in (P2R, P2C))
        assert tuple(q[1 + n0].tolist()) == (P3P1, 0, 1, 1)


@pytest.mark.parametrize("split,nb", [(1, 5), (2, 2), (2, 7), (2, 16), (4, 3), (4, 16), (16, 2), (16, 9)])
def test_small_kernel_queue_split_parts(lib, monkeypatch, split, nb):
    """APSP_SMALL_SPLIT: the chain panel tiles P2R(k; k,k+1) / P2C(k; k+1,k) in 1 (whole) or 4 parts;
    the queue still holds every task once and drains under the kernel's waits."""
    monkeypatch.setenv("APSP_SMALL_SPLIT", str(split))
    q = lib.apsp_debug_queue(nb, -1, 0, 0)
    assert sorted(expand_fused(q)) == sorted(expected_tasks(nb))
    assert len(q) == nb ** 3 - (nb - 1) + 2 * (split - 1) * (nb - 1)
    assert sum(1 for t in q.tolist() if t[0] >= 1 << PART_SHIFT) == (2 * split * (nb - 1) if split > 1 else 0)
    assert simulate(nb, [q])


def test_simulator_rejects_fused_entry_before_a_part(lib):
    """Pin of the split rule: F(0) ahead of the last part of the column-panel tile it reads cannot drain."""
    q = lib.apsp_debug_queue(6, -1, 0, 0).tolist()
    f = next(x for x, t in enumerate(q) if t[0] == P3P1 and t[1] == 0)
    last = max(x for x, t in enumerate(q) if t[0] >= 1 << PART_SHIFT and t[0] & 15 == P2C and t[1] == 0)
    q.insert(f, q.pop(last))  # the part now sits right behind F(0)
    assert not simulate(6, [np.array(q)])


def test_simulator_rejects_fused_entry_before_its_panels(lib):
    """Pin of the fused-entry rule: F(0) moved ahead of the panel tiles it reads cannot drain."""
    q = lib.apsp_debug_queue(6, -1, 0, 0).tolist()
    f = next(x for x, t in enumerate(q) if t[0] == P3P1 and t[1] == 0)
    q.insert(1, q.pop(f))
    assert not simulate(6, [np.array(q)])


@pytest.mark.parametrize("nb,delay", [(1, 0), (2, 0), (3, 0), (4, 0), (5, 3), (6, 8), (7, 100), (8, 1184), (16, 40),
                                      (33, 5), (70, 1184), (131, 592)])
def test_pair_queue_complete_and_deadlock_free(lib, nb, delay):
    """The single-GPU kernel's two-round schedule (decode2): tiles off rows / columns k, k+1 get
    rounds k and k+1 in one task; panel copies are kept for 4 rounds. Every task of the blocked FW
    exactly once and an in-order drain under the exact waits (4-parity reuse rule), including the
    multi-band phase 3 (nb >= 67) and odd nb (a last single round)."""
    q = lib.apsp_debug_queue(nb, -2, 0, delay)
    assert sorted(expand_fused(q)) == sorted(expected_tasks(nb))
    n_pairs = sum(1 for t in q.tolist() if t[0] == PAIR)
    assert n_pairs == (nb // 2) * (nb - 2) ** 2 if nb >= 2 else n_pairs == 0
    assert simulate(nb, [q], par=4)


def test_pair_queue_needs_four_parities(lib):
    """Pin of the parity rule: with only two panel-copy parities the pair queue cannot drain
    (round k+2's panels would overwrite copies the pairs of (k, k+1) still read)."""
    q = lib.apsp_debug_queue(12, -2, 0, 40)
    assert simulate(12, [q], par=4)
    assert not simulate(12, [q], par=2)
