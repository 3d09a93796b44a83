"""Multi-process (world_size 2 and 4, gloo on CPU) check of the N>1 host logic: the Ulysses
all-to-all plans exported by libtsv.so (tsv_a2a_plan — the same plans the NCCL path issues as
ncclSend/ncclRecv) executed with real point-to-point messages between processes, against the
oracle's simulated Ulysses layout (oracle/sp.py), plus the reshard plan between two groups."""
import os
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")
import torch.distributed as dist  # noqa: E402
import torch.multiprocessing as mp  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _exchange(ops, k, rank, sendbuf, recvbuf, w):
    """Execute a plan with gloo isend/irecv; the j-th op with a peer carries tag j on both sides."""
    reqs, nth = [], {}
    local_sends = [o for o in ops if o[0] == rank and o[1] == 1]
    local_recvs = [o for o in ops if o[0] == rank and o[1] == 0]
    for (_, _, s0, n), (_, _, r0, n2) in zip(local_sends, local_recvs):
        assert n == n2
        recvbuf[r0 * w:(r0 + n) * w] = sendbuf[s0 * w:(s0 + n) * w]
    for peer, is_send, row0, rows in ops:
        if peer == rank:
            continue
        key = (peer, is_send)
        tag = nth.get(key, 0)
        nth[key] = tag + 1
        if is_send:
            reqs.append(dist.isend(sendbuf[row0 * w:(row0 + rows) * w].contiguous(), peer, tag=tag))
        else:
            buf = torch.empty(rows * w, dtype=sendbuf.dtype)
            reqs.append((dist.irecv(buf, peer, tag=tag), buf, row0))
    for r in reqs:
        if isinstance(r, tuple):
            r[0].wait()
            recvbuf[r[2] * w:r[2] * w + r[1].numel()] = r[1]
        else:
            r.wait()


def _worker(rank, k, port, Lt, Li, H, D, errq):
    try:
        import sys
        sys.path.insert(0, ROOT)
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
        dist.init_process_group("gloo", rank=rank, world_size=k)
        import paper_conf_asplos_luhtlwm0c26_b200 as tsv
        from oracle import sp as SP
        L = Lt + Li
        g = np.arange(L * 3 * H * D, dtype=np.float64).reshape(L, 3, H, D)   # global joint qkv, rows [txt; img]
        t0, t1 = SP.shard_range(Lt, k, rank)
        i0, i1 = SP.shard_range(Li, k, rank)
        local = np.concatenate([g[t0:t1], g[Lt + i0:Lt + i1]])              # [rows_r, 3, H, D]
        rows_r, hk = local.shape[0], H // k
        # pack [k][rows_r][3][H/k][D] (what the fused QKV epilogue writes)
        pack = np.stack([local[:, :, d * hk:(d + 1) * hk] for d in range(k)])
        w1 = 3 * hk * D
        send = torch.from_numpy(pack.reshape(-1).copy())
        recv = torch.full((L * w1,), -1.0, dtype=torch.float64)
        _exchange(tsv.a2a_plan(1, Lt, Li, k, rank), k, rank, send, recv, w1)
        got = recv.numpy().reshape(L, 3, hk, D)
        # oracle: rank d holds heads [d*hk, (d+1)*hk) of all rows in global order (= k=1 order)
        qs_t = [g[slice(*SP.shard_range(Lt, k, r))] for r in range(k)]
        qs_i = [g[Lt:][slice(*SP.shard_range(Li, k, r))] for r in range(k)]
        ref = np.concatenate([np.concatenate(qs_t), np.concatenate(qs_i)])[:, :, rank * hk:(rank + 1) * hk]
        assert np.array_equal(got, ref), "a2a #1 layout"
        # a2a #2: attention output O (take the q part as stand-in) [L][H/k*D] back to token shards
        o = torch.from_numpy(got[:, 0].reshape(-1).copy())
        w2 = hk * D
        orecv = torch.full((k * rows_r * w2,), -1.0, dtype=torch.float64)
        _exchange(tsv.a2a_plan(2, Lt, Li, k, rank), k, rank, o, orecv, w2)
        back = orecv.numpy().reshape(k, rows_r, hk, D).transpose(1, 0, 2, 3).reshape(rows_r, H, D)
        assert np.array_equal(back, local[:, 0]), "a2a #2 inverse"
        dist.barrier()
        dist.destroy_process_group()
    except Exception as ex:  # pragma: no cover - reported to the parent
        import traceback
        errq.put(f"rank {rank}: {ex!r}\n{traceback.format_exc()}")


@pytest.mark.parametrize("k,Lt,Li", [(2, 64, 256), (4, 66, 195), (4, 512, 1024)])
def test_a2a_plans_gloo(k, Lt, Li):
    ctx = mp.get_context("spawn")
    errq = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, k, port, Lt, Li, 4, 2, errq)) for r in range(k)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(300)
    errs = []
    while not errq.empty():
        errs.append(errq.get())
    assert not errs, "\n".join(errs)
    assert all(p.exitcode == 0 for p in procs), [p.exitcode for p in procs]


def test_a2a_plan_counts():
    import paper_conf_asplos_luhtlwm0c26_b200 as tsv
    for k in (1, 2, 4, 8):
        for r in range(k):
            p1 = tsv.a2a_plan(1, 512, 16384, k, r)
            p2 = tsv.a2a_plan(2, 512, 16384, k, r)
            # every rank sends its own rows to every peer and receives every peer's rows
            assert sum(o[3] for o in p1 if o[1]) == k * (SP_rows(512, k, r) + SP_rows(16384, k, r))
            assert sum(o[3] for o in p1 if not o[1]) == 512 + 16384
            assert sum(o[3] for o in p2 if o[1]) == 512 + 16384
            assert sum(o[3] for o in p2 if not o[1]) == k * (SP_rows(512, k, r) + SP_rows(16384, k, r))


def SP_rows(n, k, r):
    from oracle import sp as SP
    a, b = SP.shard_range(n, k, r)
    return b - a
