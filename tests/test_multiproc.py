"""N > 1 host plumbing on CPU with torch.distributed gloo, world_size 2 (no GPU needed).

Covers what every rank of a multi-GPU run does before the count allreduce:
* the ncclUniqueId created by rank 0 reaches every rank through torch.distributed (distributed_nccl_id);
* every rank derives the same unit sharding from the same batch (gcsm_shard, LPT) and the shards are a disjoint
  cover of the level-1 units;
* the per-rank counts of the units a rank owns sum to the whole batch's counts (oracle IVM per unit shard),
  i.e. a sum-allreduce of the rank counters is exact.
"""
import os
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")
import torch.distributed as dist  # noqa: E402
import torch.multiprocessing as mp  # noqa: E402


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, out_q):
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    sys.path.insert(0, root)
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import gcsm_inputs as gi
        import oracle
        import paper_conf_ipps_wei024_b200 as G
        nid = G.distributed_nccl_id()
        ids = [None] * world
        dist.all_gather_object(ids, nid)
        # the same batch on every rank -> the same units and costs -> the same shard map
        w = gi.make_workload("C2", scale=10, n_edges=6000, batch=128, n_batches=1)
        ins, dele = w.batches[0]
        k, qe, ql = gi.query("diamond")
        I, D, _ = oracle.normalize_batch(w.n, w.row_ptr, w.col, ins, dele)
        U = oracle.units(k, qe, ql, None, I, D)
        deg = np.diff(w.row_ptr)
        cost = (1 + deg[U[:, 2]] + deg[U[:, 3]]).astype(np.uint64)
        ranks = G.shard(cost, world)
        maps = [None] * world
        dist.all_gather_object(maps, ranks.tolist())
        mine = set(np.nonzero(ranks == rank)[0].tolist())
        # this rank's counts: the oracle's IVM loops over its own units only
        keep = np.zeros(len(U), bool)
        keep[sorted(mine)] = True
        U_all = U

        def unit_filter(Ux):
            assert np.array_equal(Ux, U_all)
            return keep

        r = oracle._ivm(0, w.n, w.row_ptr, w.col, None, k, qe, ql, ins, dele, unit_filter=unit_filter)
        t = torch.tensor([r["added"], r["removed"]], dtype=torch.int64)
        dist.all_reduce(t)  # the count allreduce (gloo here, NCCL on the GPUs)
        full = oracle.delta(w.n, w.row_ptr, w.col, None, k, qe, ql, ins, dele)
        out_q.put((rank, nid, ids, maps, sorted(mine), tuple(t.tolist()), full, len(U)))
    finally:
        dist.destroy_process_group()


def test_gloo_world2_shard_and_allreduce():
    import __graft_entry__
    __graft_entry__.build()
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    res.sort()
    nid0 = res[0][1]
    assert len(nid0) == 128
    for rank, nid, ids, maps, mine, tot, full, n_units in res:
        assert all(x == nid0 for x in ids)            # rank 0's id reached everyone
        assert maps[0] == maps[1]                      # identical shard maps on every rank
        assert tot == full                             # allreduce of shard counts == whole-batch counts
    a, b = set(res[0][4]), set(res[1][4])
    assert not (a & b) and len(a | b) == res[0][7]     # disjoint cover of the units
    assert a and b                                     # both ranks got work


def _lib_worker(rank, world, port, out_q):
    """One rank of an emulated world on cuda:0: ITS OWN libgcsm context (rank, world, shard-local counts), the
    count allreduce over gloo; rank 0 checks the sums against the oracle."""
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    sys.path.insert(0, root)
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import gcsm_inputs as gi
        import oracle
        import paper_conf_ipps_wei024_b200 as G
        torch.cuda.set_device(0)
        w = gi.make_workload("C2", scale=12, n_edges=30_000, batch=256, n_batches=3)
        queries = ["diamond", "k4", "house5u"]
        g = G.Gcsm(w.n, w.row_ptr, w.col, device=0, rank=rank, world=world, local_counts=True)
        for i, q in enumerate(queries):
            k, qe, ql = gi.query(q)
            (g.set_query if i == 0 else g.add_query)(k, qe, ql)
        g.set_cache_budget(w.adj_bytes // 10)
        got, mine = [], []
        for ins, dele in w.batches:
            g.apply_batch(ins, dele)
            c = [g.query_counts(i) for i in range(len(queries))]
            mine.append(c)
            t = torch.tensor(c, dtype=torch.int64)
            dist.all_reduce(t)
            got.append([tuple(x) for x in t.tolist()])
        g.close()
        want = None
        if rank == 0:
            want, rp, col = [], w.row_ptr, w.col
            for ins, dele in w.batches:
                want.append([oracle.delta(w.n, rp, col, None, *gi.query(q), ins, dele) for q in queries])
                I, D, _ = oracle.normalize_batch(w.n, rp, col, ins, dele)
                rp, col = oracle.apply_batch(w.n, rp, col, I, D)
        out_q.put((rank, got, mine, want))
    finally:
        dist.destroy_process_group()


@pytest.mark.gpu
def test_libgcsm_world2_gloo():
    """N > 1 through the library itself (not the oracle's IVM): two processes, each its own context on cuda:0 with
    rank / world = 2, shard-local counts summed by a gloo allreduce, equal to the oracle on every batch and query;
    both ranks did work."""
    if not torch.cuda.is_available():
        pytest.skip("needs a GPU")
    import __graft_entry__
    __graft_entry__.build()
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_lib_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted([q.get(timeout=600) for _ in range(world)], key=lambda x: x[0])
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    want = res[0][3]
    for rank, got, mine, _ in res:
        assert got == want
    assert any(any(a or r for a, r in b) for b in res[0][2]) and any(any(a or r for a, r in b) for b in res[1][2])


def _shared_worker(rank, world, port, out_q, pipelined, link=False):
    """One rank of an emulated world on cuda:0 over ONE node-shared host store (gcsm_options.store_*): rank 0
    builds the store from the CSR, the others attach by handle (no CSR of their own); per-rank shard counts are
    summed over gloo; every rank exports G_{t+1} from the shared store at the end."""
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    sys.path.insert(0, root)
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import gcsm_inputs as gi
        import oracle
        import paper_conf_ipps_wei024_b200 as G
        torch.cuda.set_device(0)
        w = gi.make_workload("C2", scale=12, n_edges=30_000, batch=256, n_batches=5)
        queries = ["diamond", "k4", "house5u"]
        if rank == 0:
            g = G.Gcsm(w.n, w.row_ptr, w.col, device=0, rank=rank, world=world, local_counts=True,
                       store_rank=0, store_world=world)
            h = [g.store_handle()]
        else:
            h = [None]
        dist.broadcast_object_list(h, src=0)
        if rank > 0:
            g = G.Gcsm(w.n, None, None, device=0, rank=rank, world=world, local_counts=True,
                       store_rank=rank, store_world=world, store_handle=h[0])
        dist.barrier()
        for i, q in enumerate(queries):
            k, qe, ql = gi.query(q)
            (g.set_query if i == 0 else g.add_query)(k, qe, ql)
        g.set_cache_budget(w.adj_bytes // 10)
        if link:
            g.link_store_peers()
        mine, peer = [], []

        def collect():
            g.wait_batch()
            mine.append([g.query_counts(i) for i in range(len(queries))])
            peer.append(sum(g.query_stats(i)["peer_bytes"] for i in range(len(queries))))

        for b, (ins, dele) in enumerate(w.batches):
            if pipelined:
                g.submit_batch(ins, dele)
                if b >= 1:
                    collect()
            else:
                g.apply_batch(ins, dele)
                mine.append([g.query_counts(i) for i in range(len(queries))])
                peer.append(sum(g.query_stats(i)["peer_bytes"] for i in range(len(queries))))
        if pipelined:
            collect()
        got = []
        for c in mine:
            t = torch.tensor(c, dtype=torch.int64)
            dist.all_reduce(t)
            got.append([tuple(x) for x in t.tolist()])
        rp_f, col_f = g.export_csr()
        dist.barrier()  # nobody unmaps the store before every rank exported it
        g.close()
        want = rp_w = col_w = None
        if rank == 0:
            want, rp, col = [], w.row_ptr, w.col
            for ins, dele in w.batches:
                want.append([oracle.delta(w.n, rp, col, None, *gi.query(q), ins, dele) for q in queries])
                I, D, _ = oracle.normalize_batch(w.n, rp, col, ins, dele)
                rp, col = oracle.apply_batch(w.n, rp, col, I, D)
            rp_w, col_w = rp, col
        out_q.put((rank, got, mine, want, rp_f, col_f, rp_w, col_w, sum(peer)))
    finally:
        dist.destroy_process_group()


@pytest.mark.gpu
@pytest.mark.parametrize("world,pipelined,link", [(2, False, False), (3, True, False), (2, True, True),
                                                  (3, False, True)])
def test_shared_store_world_gloo(world, pipelined, link):
    """Node-shared host store: R processes on cuda:0, ONE pinned store created by rank 0
    and attached by the others; each rank writes the overlays / merges of the updated vertices it owns. Shard counts
    summed over gloo equal the oracle on every batch and query, and every rank exports the oracle's final graph
    from the shared store (so the owner-partitioned merges composed into G_{t+1}). With `link` the ranks also read
    each other's HBM caches through CUDA IPC (gcsm_link_store_peers, NEXT-3 across processes): counts unchanged and
    some list bytes served by a peer."""
    if not torch.cuda.is_available():
        pytest.skip("needs a GPU")
    import __graft_entry__
    __graft_entry__.build()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_shared_worker, args=(r, world, port, q, pipelined, link)) for r in range(world)]
    for p in procs:
        p.start()
    res = sorted([q.get(timeout=600) for _ in range(world)], key=lambda x: x[0])
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    want, rp_w, col_w = res[0][3], res[0][6], res[0][7]
    for rank, got, mine, _, rp_f, col_f, _, _, _ in res:
        assert got == want
        assert np.array_equal(rp_f, rp_w) and np.array_equal(col_f, col_w)
        assert any(any(a or r for a, r in b) for b in mine)
    peer_bytes = sum(x[8] for x in res)
    assert (peer_bytes > 0) if link else (peer_bytes == 0)
