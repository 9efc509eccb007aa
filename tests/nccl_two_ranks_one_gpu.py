"""(Round-1 diagnostic, kept under tests/ because it calls the oracle; NCCL refuses two ranks on one
GPU, profiles/r01s2_nccl_two_ranks_one_gpu.log -- the loopback tests replace it.)
Exercise the library's NCCL halo path with 2 ranks on ONE GPU (if NCCL allows it):
gloo broadcasts the ncclUniqueId, each rank owns one block, and the filled state must
equal the oracle's global fill bit for bit; then RK steps are compared with the oracle."""
import os, sys, json
sys.path.insert(0, os.getcwd()); sys.path.insert(0, os.path.join(os.getcwd(), "tests"))
import numpy as np
import torch
import torch.distributed as dist

def main():
    rank = int(os.environ["RANK"]); world = int(os.environ["WORLD_SIZE"])
    dist.init_process_group("gloo")
    import oracle, synth
    from _harness import Problem, block_slices, inner, rel_linf, state_scale
    from paper_conf_ipps_davissngmb23_b200 import crocco as cc
    from paper_conf_ipps_davissngmb23_b200.solver import Solver
    torch.cuda.set_device(0)
    uid = torch.zeros(128, dtype=torch.uint8)
    if rank == 0:
        uid.copy_(torch.frombuffer(bytearray(cc.crocco_nccl_unique_id()), dtype=torch.uint8))
    dist.broadcast(uid, 0)
    n, nb = (32, 24, 16), (2, 1, 1)
    g = synth.Wavy3D(L=(10.0,) * 3, N=n)
    pb = Problem(n, g, ((0, 0),) * 3, synth.random_state(n, seed=3), dict(terms=3, mu_ref=0.02))
    _, met, Uref = pb.oracle_inputs()
    bn, blocks = block_slices(n, nb)
    res = {"rank": rank}
    try:
        S = Solver(n, nb, pb.bc, cc.make_phys(terms=3, mu_ref=0.02), rank=rank, nranks=world,
                   block_rank=[0, 1], nccl_unique_id=bytes(uid.numpy().tobytes()))
        b = rank
        o, sl = blocks[b]
        S.set_coords([g.coords(bn, o, oracle.GC)])
        S.set_state([np.ascontiguousarray(pb.U0[(slice(None),) + sl])])
        S.fill()
        S.sync()
        got = S.view(S.U[0], 0, 5).cpu().numpy()
        ref = Uref[:, :, :, o[0]:o[0] + bn[0] + 8]
        res["fill_bitwise"] = bool(np.array_equal(got, ref))
        U = Uref.copy()
        oracle.advance(n, pb.bc, pb.oracle_phys(), 1e-3, 3, U, met)
        S.step(1e-3, 3)
        S.sync()
        gotU = S.view(S.U[0], 0, 5).cpu().numpy()[:, 4:-4, 4:-4, 4:-4]
        refU = U[:, 4:-4, 4:-4, 4 + o[0]:4 + o[0] + bn[0]]
        res["rk3_rel_err"] = rel_linf(gotU, refU, state_scale(refU))
        res["dt"] = S.compute_dt(0.5)
        S.close()
    except Exception as e:
        res["error"] = repr(e)
    print(json.dumps(res), flush=True)
    dist.barrier()

main()
