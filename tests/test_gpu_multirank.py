"""Multi-rank path on ONE GPU: 2, 4 and 8 processes share the device, exchange panel
tiles through same-device CUDA IPC peer memory (the code path NVLink peers use on a multi-GPU
box), 2D block-cyclic ownership P x Q (1x2, 2x2 and the C4 grid 2x4).  Every rank must return the
same l; it must match the CPU oracle (FP64 definition: l <= 1e-10; adaptive map: maps bit-exact
against the oracle's, l <= 1e-8 vs the FP64 oracle) and the single-rank GPU result."""
import os
import socket

import numpy as np
import pytest

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, P, Q, port, n, nb, theta, mode, q):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    import torch.distributed as dist
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_cluster_caoalgkb23_b200 as mp
        import synth
        x, y = synth.locations(n, 0)
        z = synth.normal_vector(n, 1)
        h = mp.Handle(0, rank, world, P, Q, uid=mp.shared_unique_id())
        ev = mp.Evaluator(n, nb, handle=h)
        out = []
        for md in mode:
            rep = ev.eval(x, y, z, theta, mode=md)
            km, _, cm = ev.M.maps()
            out.append((rep.loglik, rep.logdet, rep.quad, list(rep.tiles), km.tobytes(), cm.tobytes()))
        q.put((rank, out, None))
    except Exception as e:  # pragma: no cover - reported to the parent
        import traceback
        q.put((rank, None, traceback.format_exc()))
    finally:
        dist.destroy_process_group()


def run_ranks(world, P, Q, n, nb, theta, modes):
    import torch.multiprocessing as tmp
    ctx = tmp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, P, Q, port, n, nb, theta, modes, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = {}
    for _ in range(world):
        r, out, err = q.get(timeout=900)
        assert err is None, err
        res[r] = out
    for p in procs:
        p.join(timeout=60)
    return res


@pytest.fixture(scope="module")
def oracle_ref():
    """The oracle's FP64 l and maps for the shared workload (n = 4096, nb = 512, NT = 8)."""
    import synth
    from oracle.loglik import loglik as oracle_loglik
    from oracle.precision import precision_maps
    from oracle.tiles import num_tiles, tile_sqnorms
    from tests.gpu_helpers import near_tie_guard
    n, nb, theta = 4096, 512, (1.0, 0.03, 0.5)
    x, y = synth.locations(n, 0)
    z = synth.normal_vector(n, 1)
    ref = oracle_loglik(x, y, z, theta, nb)
    nt = num_tiles(n, nb)
    s = tile_sqnorms(ref["tiles"], nt)
    near_tie_guard(s, nt, 1e-9)
    km, _, cm = precision_maps(s, 1e-9)
    return {"n": n, "nb": nb, "theta": theta, "ll": ref["loglik"], "km": km, "cm": cm}


@pytest.mark.parametrize("world,P,Q", [(2, 1, 2), (4, 2, 2), (8, 2, 4)])
def test_multirank_matches_oracle_and_single_rank(world, P, Q, oracle_ref):
    import paper_conf_cluster_caoalgkb23_b200 as mp
    import synth
    n, nb, theta = oracle_ref["n"], oracle_ref["nb"], oracle_ref["theta"]
    modes = [mp.MP_MAP_ADAPTIVE, mp.MP_MAP_FP64]
    x, y = synth.locations(n, 0)
    z = synth.normal_vector(n, 1)
    ev = mp.Evaluator(n, nb)
    single = [ev.eval(x, y, z, theta, mode=md) for md in modes]
    res = run_ranks(world, P, Q, n, nb, theta, modes)
    ll_ref = oracle_ref["ll"]
    nt = ev.nt
    for i, ref in enumerate(single):
        vals = [res[r][i] for r in range(world)]
        for v in vals[1:]:
            assert v[0] == vals[0][0] and v[1] == vals[0][1]  # identical on every rank
        ll = vals[0][0]
        if modes[i] == mp.MP_MAP_FP64:
            assert abs(ll - ll_ref) <= 1e-10 * abs(ll_ref)
        else:  # maps bit-exact vs the oracle's (same on every rank), l vs the FP64 definition
            km = np.frombuffer(vals[0][4], np.uint8).reshape(nt, nt)
            cm = np.frombuffer(vals[0][5], np.uint8).reshape(nt, nt)
            low = np.tril(np.ones((nt, nt), bool))
            assert np.array_equal(km[low], oracle_ref["km"][low])
            assert np.array_equal(cm[low], oracle_ref["cm"][low])
            assert abs(ll - ll_ref) <= 1e-8 * abs(ll_ref)
        assert abs(ll - ref.loglik) <= 1e-12 * abs(ref.loglik)  # vs the single-rank GPU result
