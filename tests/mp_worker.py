"""Multi-process worker (one process per GPU slot), launched by torchrun from
tests/test_gpu_mp.py.  Each rank owns slot `rank` of a p x q grid, holds only
its own tiles and runs only its own tasks (stf_mp_*); tiles cross processes
through CUDA IPC replicas + device-side flags.  Rank 0 then re-factors the same
matrix in single-process mode with virtual slots and checks bit equality.

argv: n nb p q [push] [reps] [graph] [p2]
With p2 = 1 the input is the P2 dyadic matrix A = L0 L0^T and
every rank's tiles must also equal L0 bit for bit.
"""
import os
import sys

import numpy as np
import torch
import torch.distributed as dist

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_augonnetasg24_b200 as stf  # noqa: E402


def main():
    n, nb, p, q = (int(a) for a in sys.argv[1:5])
    push = int(sys.argv[5]) if len(sys.argv) > 5 else 0
    reps = int(sys.argv[6]) if len(sys.argv) > 6 else 2
    graph = int(sys.argv[7]) if len(sys.argv) > 7 else 1
    p2 = int(sys.argv[8]) if len(sys.argv) > 8 else 0
    dist.init_process_group("gloo")
    rank, world = dist.get_rank(), dist.get_world_size()
    assert world == p * q
    dev = int(os.environ.get("STF_MP_DEVICE", "0"))
    torch.cuda.set_device(dev)
    seed = 20240917
    stf.mp_init(rank, world, dev)
    stf.set_option("push", push)
    stf.set_option("graph", graph)
    A = stf.MpTiledMatrix(n, nb, p, q, rank, dev)
    blob = A.prepare()
    blobs = [None] * world
    dist.all_gather_object(blobs, blob)
    A.import_blobs(blobs)
    if p2:
        import synth
        Ad, L0 = synth.dyadic_spd(101, n)

    def fill():
        if not p2:
            A.fill_spd(seed)
            return
        for (i, j), t in A.tiles.items():
            t.copy_(torch.from_numpy(np.ascontiguousarray(Ad[i * nb:(i + 1) * nb, j * nb:(j + 1) * nb].T)))

    infos, times = [], []
    for _ in range(reps):  # re-run the same plan: each run clears its flags at the end
        fill()
        torch.cuda.synchronize()
        dist.barrier()
        infos.append(A.potrf())
        st = stf.last_stats()
        times.append(st["device_ms"])
        dist.barrier()
    mine = {ij: t.T.cpu().numpy().copy() for ij, t in A.tiles.items()}
    p2_bad = 0
    if p2:
        for (i, j), blk in mine.items():
            ref = L0[i * nb:(i + 1) * nb, j * nb:(j + 1) * nb]
            if i == j:
                blk, ref = np.tril(blk), np.tril(ref)
            p2_bad += not np.array_equal(blk, ref)
    assert p2_bad == 0, "rank %d: %d tiles differ from L0" % (rank, p2_bad)
    allt = [None] * world
    dist.all_gather_object(allt, (mine, infos, times, st["graph_nodes"]))
    dist.barrier()
    stf.finalize()
    if rank == 0:
        stf.init(world, [dev] * world)
        stf.set_option("push", push)
        R = stf.TiledMatrix(n, nb, p, q, devices=[dev] * world)
        if p2:
            R.load_dense(torch.from_numpy(np.ascontiguousarray(Ad)))
        else:
            R.fill_spd(seed)
        info_ref = R.potrf()
        stf.finalize()
        bad = 0
        for (m, inf, _tm, _g) in allt:
            assert all(i == info_ref for i in inf), (inf, info_ref)
            for (i, j), blk in m.items():
                ref = R.tiles[(i, j)].T.cpu().numpy()
                if not np.array_equal(blk, ref):
                    bad += 1
        ntiles = sum(len(m) for m, _, _, _ in allt)
        assert ntiles == (n // nb) * (n // nb + 1) // 2
        print("MP_RESULT world=%d tiles=%d mismatched=%d info=%d p2=%d graph_nodes=%s ms=%s" %
              (world, ntiles, bad, info_ref, p2, [g for _, _, _, g in allt], [round(x, 3) for _, _, t, _ in allt for x in t]))
        assert bad == 0
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
