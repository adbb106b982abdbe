"""Multi-rank flow of the library on one GPU: two processes, both on
cuda:0, a gloo process group with CUDA tensors (this pool gives one GPU per call; NCCL needs one
GPU per rank). Each rank detects its kernel range, histograms its sample shard, the histograms are
reduce-scattered by the kernel-aligned slot ranges, each rank joins and ranks its own sites against
its summed slice (gs_rank_sites_slice), and the exact global ranking is the merge of the ranks'
lists under the total order R20 (dist.gather_ranked). The merged R lines and every rank's K/S lines
equal the single-process oracle's."""
import os
import socket

import numpy as np
import pytest

import oracle_run as orc
from oracle_run import Canon

pytestmark = [pytest.mark.gpu, pytest.mark.usefixtures("oracle_bin")]


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, cfg, n, order, mode, row, outdir):
    import torch
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    import paper_conf_sc_senvs23_b200 as g
    from paper_conf_sc_senvs23_b200 import dist as gdist, report
    from gen import samples as gsm
    from gen import sass as gsass
    from gen.device import DeviceTrace
    s = gsass.config_sass(cfg, scale=0.004) if cfg == "C3" else gsass.config_sass(cfg)
    tab = gsm.table_class_weighted(s.cls, n, key=5)
    tr = gsm.Trace(tab, s.first_slot, s.n_instr, order=order, seed=5)
    a, b = gdist.sample_range(tr.N, rank, world)
    kb, ke = gdist.kernel_range(s.n_instr, rank, world)
    ranges = gdist.slot_ranges(s.first_slot, s.n_instr, world)
    s0, s1 = ranges[rank]
    words = DeviceTrace(tr, 0).packed(a, b)
    ctx = g.Context(device=0, n_reasons=19, hist_mode=mode, hist_row=row)
    ctx.load_sass(s.text)
    ctx.detect(kb, ke)
    hist = torch.empty(ctx.n_instr * row, dtype=torch.int32, device="cuda")
    ninv = torch.zeros(1, dtype=torch.int64, device="cuda")
    ctx.attribute_samples(words, hist, ninv)
    part = gdist.reduce_scatter_hist(hist, row, ranges)
    rows = ctx.rank_sites(part, k=None, slot_begin=s0, slot_end=s1)
    merged = gdist.gather_ranked(rows, None)
    canon = report.canonical(ctx, kb, ke)
    with open(os.path.join(outdir, f"rank{rank}.txt"), "w") as f:
        f.write(canon)
    if rank == 0:
        R = 19
        lines = [f"R {q} {int(r['kernel'])} {int(r['idx'])} {g.RULES[r['rule']]} rel={int(r['rel'])} "
                 f"tot={int(r['tot'])} ktot={int(r['ktot'])} h=" + ",".join(str(int(x)) for x in r["counts"][:R])
                 for q, r in enumerate(merged)]
        with open(os.path.join(outdir, "merged.txt"), "w") as f:
            f.write("\n".join(lines) + "\n")
        np.save(os.path.join(outdir, "raw.npy"), tr.raw())
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,cfg,n,order,mode,row", [
    (2, "C2", 2_000_000, "trace", 0, 19),
    (2, "C2", 2_000_000, "shuffled", 4, 19),
    (3, "C3", 1_000_000, "trace", 0, 32),
])
def test_multirank_flow_equals_oracle(tmp_path, world, cfg, n, order, mode, row):
    import torch.multiprocessing as mp
    from gen import sass as gsass
    port = _free_port()
    mp.start_processes(_worker, args=(world, port, cfg, n, order, mode, row, str(tmp_path)), nprocs=world,
                       start_method="spawn", join=True)
    s = gsass.config_sass(cfg, scale=0.004) if cfg == "C3" else gsass.config_sass(cfg)
    raw = np.load(tmp_path / "raw.npy")
    want = Canon(orc.run(s.text, samples=raw))
    K, S = [], []
    for r in range(world):
        c = Canon((tmp_path / f"rank{r}.txt").read_text())
        K += c.K
        S += c.S
    assert K == want.K and S == want.S
    got_R = [ln for ln in (tmp_path / "merged.txt").read_text().splitlines() if ln]
    assert got_R == want.R
    assert len(got_R) == len(want.S)
