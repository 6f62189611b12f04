"""Model check of the fused in-kernel halo synchronisation (DESIGN.md sec. 8,
kernels_vi2.cuh: HaloSync, hs_gate, hs_signal) on the CPU.

The protocol cannot run across distinct GPUs here (one GPU per box), so this
test replays it on the real partition plan the library computes
(cme_matrix_plan_partition + the packed local layouts at 2, 3, 4 and 8 ranks)
under random interleavings of the ranks' tiles:

* tiles: the tile-record kernel's tiles of `ncw` slices of every rank's local
  pack; a tile is a *halo* tile if one of its rows gathers a column outside the
  rank's own rows, a *push* tile if one of its rows lies in a peer's x span
  (the same rule as device.cu: hs_plan);
* gates (hs_gate): a halo tile of step k waits for pushed[q] >= k from every
  peer q that pushes to it; a push tile of step k waits for consumed[p] >= k
  from every peer p it pushes to;
* signals (hs_signal): when a rank's last push tile of step k is done it sets
  pushed = k + 1 at its send peers; when its last halo tile of step k is done it
  sets consumed = k + 1 at its receive peers;
* a rank's step k + 1 starts when all its step-k tiles are done (the kernel
  boundary; PDL only lets the next step's constant records load early).

Every halo read must see the value the owner produced at the previous step
(RAW), and no push may overwrite a value a peer has yet to read (WAR); the run
must never deadlock.  The x buffers alternate by step parity as on the GPU.
"""
import random

import numpy as np
import pytest

import paper_conf_ipps_maggionibl13_b200 as cme
import workloads as W


def toggle70():
    s, r, c, v = cme.cme_network_enumerate(W.toggle_switch(70))
    return len(s), r, c, v, cme.CME_ORDER_RCM


def directed_ring(n=9600, hops=(1, 5)):
    """j -> j + h (mod n): row i gathers only lower columns (and the wrap), so a
    rank's halo tiles (its first rows) and push tiles (its last rows) differ."""
    j = np.arange(n)
    r = np.concatenate([(j + h) % n for h in hops]).astype(np.int32)
    c = np.concatenate([j for _ in hops]).astype(np.int32)
    v = np.concatenate([np.full(n, 1.0 / (k + 1)) for k in range(len(hops))])
    return n, r, c, v, cme.CME_ORDER_NONE


def plan_ranks(world, ncw, problem=toggle70):
    n, r, c, v, order = problem()
    ranks = []
    for rank in range(world):
        m = cme.Matrix(n, r, c, v).reorder(order)
        m.pack(device=cme.CME_DEVICE_HOST_ONLY)
        cme.cme_matrix_plan_partition(m.h, world, rank)
        H = cme.cme_export_halo(m.h)
        P = m.packed()
        m.close()
        r0, r1 = int(H["cuts"][rank]), int(H["cuts"][rank + 1])
        lo, hi = (int(x) for x in H["span"][rank])
        own_off = r0 - lo
        nl = P["n"]
        tiles = []
        n_tiles = (P["n_slices"] + ncw - 1) // ncw
        for t in range(n_tiles):
            rows, reads = [], set()
            for q in range(t * ncw, min((t + 1) * ncw, P["n_slices"])):
                for lane in range(32):
                    slot = q * 32 + lane
                    if slot >= nl:
                        continue
                    rloc = int(P["row_of"][slot]) if P["row_of"].size else slot
                    rows.append(r0 + rloc)
                    for w in range(int(P["slice_w"][q])):
                        xs = int(P["col"][P["slice_off"][q] + lane + 32 * w])
                        g = lo + xs                     # global row of the gathered column
                        if not (r0 <= g < r1):
                            reads.add(g)
                    if P["band_on"]:
                        for g in (r0 + rloc - 1, r0 + rloc + 1):
                            if 0 <= g < n and not (r0 <= g < r1):
                                reads.add(g)
            tiles.append(dict(rows=rows, reads=sorted(reads)))
        ranks.append(dict(r0=r0, r1=r1, lo=lo, hi=hi, tiles=tiles))
    # push targets: my rows inside a peer's span
    for a, ra in enumerate(ranks):
        ra["send"] = [b for b, rb in enumerate(ranks) if b != a and max(ra["r0"], rb["lo"]) < min(ra["r1"], rb["hi"])]
    for b, rb in enumerate(ranks):
        rb["recv"] = [a for a, ra in enumerate(ranks) if b in ra["send"]]
    for a, ra in enumerate(ranks):
        for t in ra["tiles"]:
            t["push"] = {b: [g for g in t["rows"] if ranks[b]["lo"] <= g < ranks[b]["hi"]] for b in ra["send"]}
            t["kind"] = (1 if t["reads"] else 0) | (2 if any(t["push"].values()) else 0)
    return ranks


def simulate(ranks, steps, seed, raw_gate=True, war_gate=True):
    """One random interleaving of `steps` steps of every rank; AssertionError on
    a RAW / WAR violation or a deadlock."""
    rng = random.Random(seed)
    P = len(ranks)
    # buf[b][parity][global row] = step token held in rank b's x-span copy
    buf = [[{g: 0 for g in range(rk["lo"], rk["hi"])}, {}] for rk in ranks]
    pushed = [[0] * P for _ in range(P)]     # pushed[b][a]: rank a's signal as seen by b
    consumed = [[0] * P for _ in range(P)]   # consumed[a][b]: rank b's signal as seen by a
    pending = {}                             # (reader, step) -> halo rows still to be read
    step = [0] * P
    todo = [list(range(len(rk["tiles"]))) for rk in ranks]
    left_push = [sum(1 for t in rk["tiles"] if t["kind"] & 2) for rk in ranks]
    left_halo = [sum(1 for t in rk["tiles"] if t["kind"] & 1) for rk in ranks]
    for b in range(P):
        pending[(b, 0)] = set(g for t in ranks[b]["tiles"] for g in t["reads"])
    executed = 0
    last = -1
    while min(step) < steps:
        ready = []
        for a in range(P):
            if step[a] >= steps:
                continue
            k = step[a]
            for ti in todo[a]:
                t = ranks[a]["tiles"][ti]
                ok = True
                if raw_gate and t["kind"] & 1:
                    ok = ok and all(pushed[a][q] >= k for q in ranks[a]["recv"])
                if war_gate and t["kind"] & 2:
                    ok = ok and all(consumed[a][p] >= k for p in ranks[a]["send"])
                if ok:
                    ready.append((a, ti))
        assert ready, f"deadlock at steps {step}"
        # bursty scheduler: mostly stay on the rank that ran last, so ranks race
        # ahead of each other as far as the gates allow
        same = [rt for rt in ready if rt[0] == last]
        a, ti = rng.choice(same if same and rng.random() < 0.9 else ready)
        last = a
        k, t = step[a], ranks[a]["tiles"][ti]
        par = k % 2
        for g in t["reads"]:   # RAW: the owner's step k-1 output (step 0: the loaded p0)
            assert buf[a][par].get(g) == k, ("RAW", a, k, g, buf[a][par].get(g))
            pending[(a, k)].discard(g)
        for g in t["rows"]:    # own rows into my next buffer
            buf[a][1 - par][g] = k + 1
        for b, rows in t["push"].items():   # WAR: peer b must have read these rows at step k-1
            for g in rows:
                if k >= 1:
                    assert g not in pending.get((b, k - 1), set()), ("WAR", a, b, k, g)
                buf[b][1 - par][g] = k + 1
        todo[a].remove(ti)
        executed += 1
        if t["kind"] & 2:
            left_push[a] -= 1
            if left_push[a] == 0:
                for b in ranks[a]["send"]:
                    pushed[b][a] = k + 1
        if t["kind"] & 1:
            left_halo[a] -= 1
            if left_halo[a] == 0:
                for q in ranks[a]["recv"]:
                    consumed[q][a] = k + 1
        if not todo[a]:   # kernel boundary: the next step of rank a
            assert not pending[(a, k)]
            step[a] += 1
            todo[a] = list(range(len(ranks[a]["tiles"])))
            left_push[a] = sum(1 for tt in ranks[a]["tiles"] if tt["kind"] & 2)
            left_halo[a] = sum(1 for tt in ranks[a]["tiles"] if tt["kind"] & 1)
            pending[(a, k + 1)] = set(g for tt in ranks[a]["tiles"] for g in tt["reads"])
    return executed


@pytest.mark.parametrize("problem", [toggle70, directed_ring], ids=["toggle70-rcm", "directed-ring"])
@pytest.mark.parametrize("world", [2, 3, 4, 8])
def test_fused_halo_sync_model(world, problem):
    ncw, steps = 16, 6
    ranks = plan_ranks(world, ncw, problem)
    for seed in range(4):
        executed = simulate(ranks, steps, seed * 100 + world)
        assert executed == steps * sum(len(rk["tiles"]) for rk in ranks)
    kinds = np.array([t["kind"] for rk in ranks for t in rk["tiles"]])
    assert (kinds & 1).any() and (kinds & 2).any()
    if problem is toggle70:   # RCM: only the boundary tiles take part, most tiles are interior
        assert (kinds == 0).mean() > 0.3


@pytest.mark.parametrize("drop", ["raw", "war"])
def test_fused_halo_sync_model_catches_a_missing_gate(drop):
    """The replay has teeth: without either gate some interleaving reads a
    stale halo row (RAW) or overwrites one a peer has not read yet (WAR).  (On
    the symmetric CME bands a boundary tile both reads and pushes halo rows, so
    each gate masks the other; the directed ring separates them.)"""
    ranks = plan_ranks(2, 16, directed_ring)
    failures = 0
    for seed in range(40):
        try:
            simulate(ranks, 4, seed, raw_gate=drop != "raw", war_gate=drop != "war")
        except AssertionError as e:   # (a missed WAR can also surface as a stale read)
            assert "'RAW'" in str(e) or "'WAR'" in str(e), str(e)
            failures += 1
    assert failures > 0
