"""Multi-rank path on ONE GPU: 2 and 4 processes share the device, exchange panel
tiles through same-device CUDA IPC peer memory (the code path NVLink peers use on a multi-GPU
box), 2D block-cyclic ownership P x Q.  Every rank must return the same l, equal to the
single-rank result (the factor is the same arithmetic; only the solve's reduction order differs)."""
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
        h = mp.Handle(0, rank, world, P, Q)
        ev = mp.Evaluator(n, nb, handle=h)
        out = []
        for md in mode:
            rep = ev.eval(x, y, z, theta, mode=md)
            out.append((rep.loglik, rep.logdet, rep.quad, list(rep.tiles)))
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


@pytest.mark.parametrize("world,P,Q", [(2, 1, 2), (4, 2, 2)])
def test_multirank_matches_single_rank(world, P, Q):
    import paper_conf_cluster_caoalgkb23_b200 as mp
    import synth
    n, nb, theta = 4096, 512, (1.0, 0.03, 0.5)
    modes = [mp.MP_MAP_ADAPTIVE, mp.MP_MAP_FP64]
    x, y = synth.locations(n, 0)
    z = synth.normal_vector(n, 1)
    ev = mp.Evaluator(n, nb)
    single = [ev.eval(x, y, z, theta, mode=md) for md in modes]
    res = run_ranks(world, P, Q, n, nb, theta, modes)
    for i, ref in enumerate(single):
        vals = [res[r][i] for r in range(world)]
        for v in vals[1:]:
            assert v[0] == vals[0][0] and v[1] == vals[0][1]  # identical on every rank
        assert vals[0][3] == list(ref.tiles)
        assert abs(vals[0][1] - ref.logdet) <= 1e-13 * abs(ref.logdet)
        assert abs(vals[0][0] - ref.loglik) <= 1e-12 * abs(ref.loglik)
