"""Multi-rank host logic on CPU (gloo, world size 2 and 4): the panel-exchange plan every rank
executes (mp_exchange_plan, the records mp_tile_potrf runs) is globally consistent, matches an
independent model of Algorithm 1's data flow on the 2D block-cyclic grid,
and works as an actual communication schedule (tiles sent over gloo arrive where they are used)."""
import os
import socket

import numpy as np
import pytest

BYTES = {0: 8, 1: 4, 2: 2}


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def owner(m, k, P, Q):
    return (m % P) * Q + (k % Q)


def needed_by(rank, k, m, nt, P, Q):
    """Independent model: does `rank` run a task that consumes L_mk (m > k) or L~_kk (m == k)?"""
    if m == k:  # TRSM(i, k) tasks, i > k
        return any(owner(i, k, P, Q) == rank for i in range(k + 1, nt))
    tasks = [(m, m)] + [(m, n) for n in range(k + 1, m)] + [(n, m) for n in range(m + 1, nt)]
    return any(owner(a, b, P, Q) == rank for a, b in tasks)


def comm_maps(nt):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    from oracle import FP16
    from oracle.precision import COMM_AUTO, COMM_TTC, comm_map, extreme_map
    rng = np.random.default_rng(nt)
    km = np.full((nt, nt), 255, np.uint8)
    for k in range(nt):
        km[k, k] = 0
        for m in range(k + 1, nt):
            km[m, k] = rng.choice([0, 1, 2], p=[0.3, 0.4, 0.3]) if m - k > 1 else 0
    ext = extreme_map(nt, FP16)
    return {"random_auto": comm_map(km, COMM_AUTO), "random_ttc": comm_map(km, COMM_TTC),
            "extreme_auto": comm_map(ext, COMM_AUTO), "extreme_ttc": comm_map(ext, COMM_TTC)}


def _worker(rank, world, P, Q, port, q):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    import torch
    import torch.distributed as dist
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_cluster_caoalgkb23_b200 import exchange_plan
        nt = 9
        result = {}
        for name, cm in comm_maps(nt).items():
            mine = exchange_plan(nt, P, Q, rank, cm)
            plans = [None] * world
            dist.all_gather_object(plans, mine)
            result[name] = plans
        # execute the plan of the "random_auto" map as a real schedule over gloo: the producer sends
        # a tile whose content encodes (k, m), every pull receives it and checks it
        cm = comm_maps(nt)["random_auto"]
        mine = exchange_plan(nt, P, Q, rank, cm)
        plans = result["random_auto"]
        ok = True
        for k in range(nt - 1):
            reqs = []
            recv = {}
            for (kk, m, peer, prec, d) in mine:
                if kk != k:
                    continue
                if d == 0:  # publish: send to every consumer that pulls it
                    payload = torch.full((16,), float(1000 * k + m))
                    for r in range(world):
                        if r != rank and any(x[:2] == (k, m) and x[4] == 1 and x[2] == rank for x in plans[r]):
                            reqs.append(dist.isend(payload, dst=r, tag=1000 * k + m))
                else:
                    buf = torch.zeros(16)
                    recv[m] = buf
                    reqs.append(dist.irecv(buf, src=peer, tag=1000 * k + m))
            for r in reqs:
                r.wait()
            for m, buf in recv.items():
                ok &= bool(torch.all(buf == float(1000 * k + m)))
        q.put((rank, result, ok, None))
    except Exception:
        import traceback
        q.put((rank, None, False, traceback.format_exc()))
    finally:
        dist.destroy_process_group()


def run(world, P, Q):
    import torch.multiprocessing as tmp
    ctx = tmp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, P, Q, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = {}
    for _ in range(world):
        r, res, ok, err = q.get(timeout=300)
        assert err is None, err
        assert ok, f"rank {r}: a pulled tile did not arrive intact"
        out[r] = res
    for p in procs:
        p.join(timeout=60)
    return out


@pytest.mark.parametrize("world,P,Q", [(2, 1, 2), (4, 2, 2)])
def test_exchange_plan_consistent_over_gloo(world, P, Q):
    out = run(world, P, Q)
    nt = 9
    maps = comm_maps(nt)
    for name, cm in maps.items():
        plans = out[0][name]
        assert all(out[r][name] == plans for r in range(world))  # every rank saw the same gather
        pubs = {(r, k, m): prec for r in range(world) for (k, m, peer, prec, d) in plans[r] if d == 0}
        pulls = [(r, k, m, peer, prec) for r in range(world) for (k, m, peer, prec, d) in plans[r] if d == 1]
        # every pull has its publish, from the tile's owner, in the comm precision of the map
        for (r, k, m, peer, prec) in pulls:
            assert peer == owner(m, k, P, Q) != r
            assert pubs[(peer, k, m)] == prec == cm[m, k]
        # every publish is pulled by someone
        for (r, k, m) in pubs:
            assert any(p[1:3] == (k, m) for p in pulls)
        # independent data-flow model: pulled = needed and not owned
        for r in range(world):
            got = {(k, m) for (k, m, peer, prec, d) in plans[r] if d == 1}
            want = {(k, m) for k in range(nt - 1) for m in range(k, nt)
                    if needed_by(r, k, m, nt, P, Q) and owner(m, k, P, Q) != r}
            assert got == want, (name, r)
    # STC halves the bytes on the extreme map (FP16 instead of the FP32 storage)
    vol = {name: sum(BYTES[prec] for r in range(world) for (k, m, peer, prec, d) in out[0][name][r]
                     if d == 1 and m > k) for name in maps}
    assert vol["extreme_auto"] * 2 == vol["extreme_ttc"]
    assert vol["random_auto"] <= vol["random_ttc"]


def _uid_worker(rank, world, port, q):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    import torch.distributed as dist
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_cluster_caoalgkb23_b200 as mp
        q.put((rank, mp.shared_unique_id(), None))
    except Exception:  # pragma: no cover - reported to the parent
        import traceback
        q.put((rank, None, traceback.format_exc()))
    finally:
        dist.destroy_process_group()


def test_communicator_id_is_shared_over_gloo():
    """mp_get_unique_id on rank 0, broadcast over torch.distributed (gloo, world size 3): every rank
    holds the same 128 bytes (the id each rank passes to mp_init_config and that mp_matrix_comm_connect
    checks in the peers' exchange areas)."""
    import torch.multiprocessing as tmp
    ctx = tmp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_uid_worker, args=(r, 3, port, q)) for r in range(3)]
    for p in procs:
        p.start()
    ids = {}
    for _ in range(3):
        r, uid, err = q.get(timeout=300)
        assert err is None, err
        ids[r] = uid
    for p in procs:
        p.join(timeout=60)
    assert len(ids[0]) == 128 and ids[0] == ids[1] == ids[2]
