"""world_size-2 multi-process test of the N>1 exchange logic on CPU (gloo).

Each rank owns some blocks of a decomposed global state; it asks libcrocco for
its exchange plan (crocco_exchange_plan, host-only), executes the plan with
numpy box copies and torch.distributed gloo send/recv in the plan's canonical
order (the order the library issues ncclSend/ncclRecv), and the stitched
result must equal the oracle's global fill bit for bit.  This pins the
message schedule and region bookkeeping of the NCCL path without a GPU.
"""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

G = 4


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, n, nb, bc, block_rank, result_q):
    import torch
    import torch.distributed as dist

    import oracle  # noqa: F401  (only to assert the same environment)
    import synth
    from paper_conf_ipps_davissngmb23_b200 import crocco as cc

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    bn = [n[d] // nb[d] for d in range(3)]
    Uglob = synth.random_state(n, seed=21)
    desc = cc.make_desc(n, nb, bc, rank=rank, nranks=world, block_rank=block_rank)
    nbt = nb[0] * nb[1] * nb[2]
    # local padded block arrays
    arrs = {}
    for b in range(nbt):
        if block_rank[b] != rank:
            continue
        bx, by, bz = b % nb[0], (b // nb[0]) % nb[1], b // (nb[0] * nb[1])
        o = (bx * bn[0], by * bn[1], bz * bn[2])
        a = np.zeros((5, bn[2] + 8, bn[1] + 8, bn[0] + 8))
        a[:, G:-G, G:-G, G:-G] = Uglob[:, o[2]:o[2] + bn[2], o[1]:o[1] + bn[1], o[0]:o[0] + bn[0]]
        arrs[b] = a

    def box(a, lo, ext):
        return a[:, lo[2] + G:lo[2] + G + ext[2], lo[1] + G:lo[1] + G + ext[1],
                 lo[0] + G:lo[0] + G + ext[0]]

    for ph in range(3):
        plan = cc.crocco_exchange_plan(desc, ph)
        # local copies and physical BCs (semantics of include/crocco.h)
        for m in plan:
            if m.dst_rank != rank or (m.kind == 0 and m.src_rank != rank):
                continue
            lo, ext = list(m.dst_lo), list(m.ext)
            dst = box(arrs[m.dst_block], lo, ext)
            if m.kind == 0:
                dst[...] = box(arrs[m.src_block], list(m.src_lo), ext)
            else:
                a = arrs[m.dst_block]
                nd = bn[ph]
                for g in range(1, G + 1):
                    di = -g if m.side == 0 else nd - 1 + g
                    if m.bc_kind == 1:
                        si = 0 if m.side == 0 else nd - 1
                        sgn = 1
                    else:  # WALL
                        si = g - 1 if m.side == 0 else nd - g
                        sgn = -1
                    l1, l2 = list(lo), list(lo)
                    e1 = list(ext)
                    l1[ph], l2[ph], e1[ph] = di, si, 1
                    v = box(a, l2, e1).copy()
                    if sgn < 0:
                        v[1:4] *= -1
                    box(a, l1, e1)[...] = v
        # remote messages in canonical order (one batch, like ncclGroupStart/End)
        reqs = []
        bufs = []
        for m in plan:
            if m.kind != 0 or m.src_rank == m.dst_rank:
                continue
            ext = list(m.ext)
            if m.src_rank == rank:
                t = torch.from_numpy(np.ascontiguousarray(box(arrs[m.src_block], list(m.src_lo), ext)))
                reqs.append(dist.isend(t, m.dst_rank))
            else:
                t = torch.empty((5, ext[2], ext[1], ext[0]), dtype=torch.float64)
                reqs.append(dist.irecv(t, m.src_rank))
                bufs.append((m, t))
        for r in reqs:
            r.wait()
        for m, t in bufs:
            box(arrs[m.dst_block], list(m.dst_lo), list(m.ext))[...] = t.numpy()
    result_q.put((rank, {b: a for b, a in arrs.items()}))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("nb,bc,block_rank", [
    ((2, 2, 1), ((0, 0),) * 3, [0, 1, 1, 0]),
    ((2, 1, 2), ((1, 1), (3, 1), (0, 0)), [0, 0, 1, 1]),
])
def test_two_rank_exchange_matches_oracle_fill(nb, bc, block_rank):
    import oracle
    import synth
    n = (16, 12, 8) if nb[2] == 1 else (16, 8, 12)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, n, nb, bc, block_rank, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = {}
    for _ in range(2):
        r, arrs = q.get(timeout=120)
        res.update(arrs)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    U = synth.pad_state(synth.random_state(n, seed=21))
    oracle.fill(n, bc, U)
    bn = [n[d] // nb[d] for d in range(3)]
    for b, a in res.items():
        bx, by, bz = b % nb[0], (b // nb[0]) % nb[1], b // (nb[0] * nb[1])
        o = (bx * bn[0], by * bn[1], bz * bn[2])
        ref = U[:, o[2]:o[2] + bn[2] + 8, o[1]:o[1] + bn[1] + 8, o[0]:o[0] + bn[0] + 8]
        assert np.array_equal(a, ref), b
