"""Worker for the multi-process tests (launched by torch.distributed.run).

mode "oracle-slabs" (CPU, gloo): the host-side distributed logic of the spread
layer on real numbers. Each rank owns the chunks of its list position of a
static round-robin spread (libsomier's host spread descriptor), steps each
chunk's slab -- owned planes plus the halo planes of map A[start-1:size+2] --
with the CPU oracle, and after every step sends its first / last owned plane
into the left / right neighbour chunk's halo (gloo send/recv when the
neighbour belongs to the other rank). Partial stats are combined exactly by
somier_stats_combine. Rank 0 gathers everything and writes it to --out.

mode "gpu-ipc" (GPU): the product path with one process per list position --
somier_init_local + CUDA IPC connect + fused in-kernel exchange -- here with
both ranks on the same physical GPU (cuda_device=0), which is the only way to
run the multi-process path on a 1-GPU box. Rank 0 writes the full state.
"""
import argparse
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402


def oracle_slabs(a):
    import oracle as O
    import paper_conf_ipps_torresft22_b200 as P
    from paper_conf_ipps_torresft22_b200 import dist as PD

    dist.init_process_group("gloo")
    rank, world = dist.get_rank(), dist.get_world_size()
    n = tuple(a.n)
    op = O.Params(n=n, seed=a.seed)
    full = O.init(op)
    spread = P.Spread(list(range(world)), 1, n[0] - 2, chunk=a.chunk)
    chunks = spread.chunks()
    mine = [c for c in chunks if c.device_pos == rank]
    slabs = {}
    for c in mine:
        f, ln = spread.map_extent(c.index, n[0], 1, 1)   # A[start-1 : size+2]
        sub = O.Params(n=(ln, n[1], n[2]), seed=a.seed)
        st = O.State(sub, *(np.ascontiguousarray(arr[f:f + ln]) for arr in
                            (full.x, full.y, full.z, full.vx, full.vy, full.vz)))
        slabs[c.index] = st
    owner = {c.index: c.device_pos for c in chunks}
    for t in range(a.steps):
        for idx in slabs:
            slabs[idx], _ = O.step(slabs[idx])
        # halo exchange: first owned plane -> left neighbour's hi halo,
        # last owned plane -> right neighbour's lo halo
        reqs, recvs = [], []
        for c in mine:
            s = slabs[c.index]
            for nb, plane, slot in ((c.index - 1, 1, "hi"), (c.index + 1, c.size, "lo")):
                if nb < 0 or nb >= len(chunks):
                    continue
                payload = np.stack([s.x[plane], s.y[plane], s.z[plane]])
                if owner[nb] == rank:
                    recvs.append((nb, slot, payload))
                else:
                    reqs.append(dist.isend(torch.from_numpy(payload.copy()), owner[nb], tag=2 * nb + (slot == "hi")))
        for c in mine:
            for nb, slot in ((c.index - 1, "lo"), (c.index + 1, "hi")):
                if nb < 0 or nb >= len(chunks) or owner[nb] == rank:
                    continue
                buf = torch.empty((3, n[1], n[2]), dtype=torch.float64)
                dist.recv(buf, owner[nb], tag=2 * c.index + (slot == "hi"))
                recvs.append((c.index, slot, buf.numpy()))
        for r in reqs:
            r.wait()
        for idx, slot, payload in recvs:
            s = slabs[idx]
            plane = 0 if slot == "lo" else s.x.shape[0] - 1
            s.x[plane], s.y[plane], s.z[plane] = payload[0], payload[1], payload[2]
    # exact partial stats of the owned planes (+ fixed end planes held as halos)
    parts = []
    for c in mine:
        s = slabs[c.index]
        lo = 0 if c.start == 1 else 1
        hi = s.x.shape[0] if c.start + c.size == n[0] - 1 else s.x.shape[0] - 1
        sub = O.State(O.Params(n=(hi - lo, n[1], n[2])),
                      *(np.ascontiguousarray(arr[lo:hi]) for arr in (s.x, s.y, s.z, s.vx, s.vy, s.vz)))
        ost = O.centers(sub)
        parts.append(P.Stats(a.steps, (0.0,) * 3, 0.0, ost.sums, ost.vmax2_bits, (hi - lo) * n[1] * n[2]))
    all_parts = [None] * world
    dist.all_gather_object(all_parts, parts)
    flat = [p for ps in all_parts for p in ps]
    st = PD.combine_partials(flat, P.SomierParams(n=n))
    owned = {c.index: np.stack([slabs[c.index].x, slabs[c.index].y, slabs[c.index].z,
                                slabs[c.index].vx, slabs[c.index].vy, slabs[c.index].vz])[:, 1:-1]
             for c in mine}
    gathered = [None] * world
    dist.all_gather_object(gathered, owned)
    if rank == 0:
        out = np.zeros((6,) + n)
        out[:3] = full.X
        for d in gathered:
            for idx, arr in d.items():
                c = chunks[idx]
                out[:, c.start:c.start + c.size] = arr
        np.savez(a.out, state=out, sums=np.array([str(v) for v in st.sums]), vmax2=np.array(str(st.vmax2_bits)),
                 centre=np.array(st.centre), nodes=np.array(st.nodes))
    dist.barrier()
    dist.destroy_process_group()


def gpu_ipc(a):
    import paper_conf_ipps_torresft22_b200 as P
    from paper_conf_ipps_torresft22_b200 import dist as PD

    dist.init_process_group("gloo")
    rank, world = dist.get_rank(), dist.get_world_size()
    torch.cuda.set_device(0)
    n = tuple(a.n)
    kernel = int(os.environ.get("SOMIER_TEST_KERNEL", P.K1_AUTO))
    exchange = int(os.environ.get("SOMIER_TEST_EXCHANGE", P.EXCHANGE_FUSED))
    params = P.SomierParams(n=n, seed=a.seed, kernel=kernel, exchange=exchange)
    s = PD.open_local(params, chunk=a.chunk, cuda_device=0)
    if kernel == P.K1_TB2:
        assert s.kernel_in_use == P.K1_TB2
    s.step(a.steps)
    s.sync()
    st = PD.gather_stats(s)
    hist = PD.gather_stats_history(s, 1, a.steps)  # every step's exact global stats
    X, V = s.read()
    mask = np.zeros(n[0], bool)
    for c in s.spread.chunks():
        if c.device_pos == rank:
            mask[c.start:c.start + c.size] = True
            if c.start == 1:
                mask[0] = True
            if c.start + c.size == n[0] - 1:
                mask[n[0] - 1] = True
    parts = [None] * world
    dist.all_gather_object(parts, (mask, X[:, mask], V[:, mask]))
    if rank == 0:
        out = np.zeros((6,) + n)
        for m, x, v in parts:
            out[:3, m] = x
            out[3:, m] = v
        np.savez(a.out, state=out, sums=np.array([str(v) for v in st.sums]), vmax2=np.array(str(st.vmax2_bits)),
                 centre=np.array(st.centre), launches=np.array(s.launches),
                 hist_sums=np.array([[str(v) for v in h.sums] for h in hist]),
                 hist_vmax2=np.array([str(h.vmax2_bits) for h in hist]))
    dist.barrier()
    s.close()
    dist.barrier()
    dist.destroy_process_group()


if __name__ == "__main__":
    # positional only: torch.distributed.run would claim option prefixes
    ap = argparse.ArgumentParser()
    for name in ("mode", "out"):
        ap.add_argument(name)
    for name in ("n0", "n1", "n2", "steps", "chunk", "seed"):
        ap.add_argument(name, type=int)
    a = ap.parse_args()
    a.n = [a.n0, a.n1, a.n2]
    {"oracle-slabs": oracle_slabs, "gpu-ipc": gpu_ipc}[a.mode](a)
