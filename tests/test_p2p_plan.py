"""Host arithmetic of one chunk of the multi-GPU exchange (cuart_dist_chunk_plan,
the plan csrc/dist.cu uses), CPU only.

The device steps are emulated with numpy: every source partitions its chunk
stably by owner (the send order of the fused K-ROUTE/K-BUCKET pass; the bucket
order inside an owner's run does not matter here), pushes run o to owner o at
push_off[o], the owner serves its window and stores the results of source s's
segment [seg_start[s], seg_start[s+1]) at res_off[s] of s's send order, and the
source gathers them back.  The plan must (i) tile every owner's receive window
with the sources' runs in rank order -- the global op order of the update rule
(reading C7) -- and (ii) bring every result back to the query it answers."""
import numpy as np
import pytest

from paper_conf_icpp_koppehelggp21_b200.dist import chunk_plan


def _emulate(batches, owner_of, f, P):
    parts = []
    M = np.zeros((P, P), np.uint64)
    for s, q in enumerate(batches):
        own = owner_of(q)
        order = np.argsort(own, kind="stable")              # send order (owner-major, stable)
        perm = np.empty(q.shape[0], np.int64)
        perm[order] = np.arange(q.shape[0])
        M[s] = np.bincount(own, minlength=P)
        parts.append((own, order, perm))
    plans = [chunk_plan(M, r) for r in range(P)]
    cap = int(M.sum(axis=0).max()) if P else 0
    win = [np.full(cap, -1, np.int64) for _ in range(P)]
    filled = [np.zeros(cap, np.int64) for _ in range(P)]
    for s, q in enumerate(batches):                         # the fused push (k_bscatter<PUSH>)
        own, order, _ = parts[s]
        sent, sent_own = q[order], own[order]
        for o in range(P):
            run = sent[sent_own == o]
            a = int(plans[s][2][o])
            win[o][a:a + run.shape[0]] = run
            filled[o][a:a + run.shape[0]] += 1
    for o in range(P):                                      # every slot written exactly once, rank order
        n = int(plans[o][0][P])
        assert n == int(M[:, o].sum())
        assert (filled[o][:n] == 1).all() and (filled[o][n:] == 0).all()
        exp = np.concatenate([q[parts[s][0] == o] for s, q in enumerate(batches)])
        assert np.array_equal(win[o][:n], exp)
    res = [np.full(max(1, q.shape[0]), -7, np.int64) for q in batches]
    for o in range(P):                                      # the owner's walk with the fused return (SegOut)
        seg, res_off, _ = plans[o]
        r = f(win[o][: int(seg[P])])
        for s in range(P):
            a, b = int(seg[s]), int(seg[s + 1])
            res[s][int(res_off[s]):int(res_off[s]) + (b - a)] = r[a:b]
    for s, q in enumerate(batches):                         # k_bgather back into query order
        assert np.array_equal(res[s][parts[s][2]], f(q))


@pytest.mark.parametrize("P", [1, 2, 3, 8, 16])
@pytest.mark.parametrize("seed", [0, 1, 2])
def test_plan_round_trip(P, seed):
    rng = np.random.default_rng(seed * 31 + P)
    sizes = rng.integers(0, 3000, P)
    sizes[rng.integers(0, P)] = 0                          # an empty source
    batches = [rng.integers(0, 1 << 40, int(m), dtype=np.int64) for m in sizes]
    skew = seed == 2
    owner_of = (lambda q: np.minimum(P - 1, (q % 7 == 0) * (q % P))) if skew else (lambda q: (q * 2654435761) % P)
    _emulate(batches, owner_of, lambda x: x * 3 + 1, P)


def test_plan_hand_example():
    M = np.array([[1, 2], [3, 4]], np.uint64)              # M[s][o]
    seg, res_off, push_off = chunk_plan(M, 1)
    assert seg.tolist() == [0, 2, 6]                       # owner 1 receives 2 from s0, then 4 from s1
    assert res_off.tolist() == [1, 3]                      # my results start after owner 0's in s's send order
    assert push_off.tolist() == [1, 2]                     # my runs land after source 0's runs
