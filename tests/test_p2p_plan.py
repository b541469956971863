"""Host arithmetic of the fused p2p exchange (dist.p2p_plan), CPU only.

The device steps are emulated with numpy (stable per-owner partition = what
cuart_route_count / cuart_route_push compute, a pure function of the key as the
owner's lookup), and the plan's offsets must (i) tile every owner's receive
window with the sources' runs in rank order — the global op order the update rule
needs (reading C7) — and (ii) bring every result back to the slot its
query came from."""
import numpy as np
import pytest

from paper_conf_icpp_koppehelggp21_b200.dist import p2p_plan


def _emulate(batches, owner_of, f, P):
    parts = []
    M = np.zeros((P, P), np.int64)
    for s, q in enumerate(batches):
        own = owner_of(q)
        order = np.argsort(own, kind="stable")              # send order (owner-major, stable)
        perm = np.empty(q.shape[0], np.int64)
        perm[order] = np.arange(q.shape[0])
        M[s] = np.bincount(own, minlength=P)
        parts.append((own, order, perm))
    plans = [p2p_plan(M, r) for r in range(P)]
    cap = plans[0]["need_recv"]
    assert all(p["need_recv"] == cap and p["need_res"] == plans[0]["need_res"] for p in plans)
    win = [np.full(cap, -1, np.int64) for _ in range(P)]
    filled = [np.zeros(cap, np.int64) for _ in range(P)]
    for s, q in enumerate(batches):                         # cuart_route_push
        own, order, _ = parts[s]
        sent = q[order]
        so = sent_own = own[order]
        for o in range(P):
            run = sent[sent_own == o]
            a = plans[s]["push_off"][o]
            win[o][a:a + run.shape[0]] = run
            filled[o][a:a + run.shape[0]] += 1
    for o in range(P):                                      # every slot written exactly once, rank order
        n = plans[o]["recv_total"]
        assert (filled[o][:n] == 1).all() and (filled[o][n:] == 0).all()
        exp = np.concatenate([q[parts[s][0] == o] for s, q in enumerate(batches)])
        assert np.array_equal(win[o][:n], exp)
    res = [np.full(plans[0]["need_res"], -7, np.int64) for _ in range(P)]
    for o in range(P):                                      # cuart_lookup_segmented
        p = plans[o]
        r = f(win[o][:p["recv_total"]])
        for s in range(P):
            a, b = p["seg_start"][s], p["seg_start"][s + 1]
            res[s][p["res_off"][s]:p["res_off"][s] + (b - a)] = r[a:b]
    for s, q in enumerate(batches):                         # cuart_unroute
        out = res[s][parts[s][2]]
        assert np.array_equal(out, f(q))


@pytest.mark.parametrize("P", [1, 2, 3, 8, 16])
@pytest.mark.parametrize("seed", [0, 1, 2])
def test_plan_round_trip(P, seed):
    rng = np.random.default_rng(seed * 31 + P)
    sizes = rng.integers(0, 5000, P)
    sizes[rng.integers(0, P)] = 0                           # an empty source
    batches = [rng.integers(0, 1 << 40, int(m)) for m in sizes]
    skew = rng.random() < 0.5
    owner_of = (lambda q: np.minimum((q >> 37) * P // 8, P - 1)) if not skew else (lambda q: np.where(q % 7 == 0, 0, (q >> 20) % P))
    _emulate(batches, owner_of, lambda x: x * 3 + 1, P)


def test_plan_hand_example():
    # 2 ranks: source 0 sends 1 op to owner 0 and 2 to owner 1; source 1 sends 3 and 4
    p1 = p2p_plan([[1, 2], [3, 4]], 1)
    assert p1["push_off"] == [1, 2]            # after source 0's runs in both owners' windows
    assert p1["seg_start"] == [0, 2, 6]        # owner 1 receives 2 then 4 ops
    assert p1["res_off"] == [1, 3]             # results go after owner 0's share at each source
    assert p1["need_recv"] == 6 and p1["need_res"] == 7
