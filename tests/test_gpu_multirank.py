"""The multi-GPU row-band path end to end through torch.distributed, with every rank on the
one GPU of the test box: world size 2 and 3 over gloo (the halo exchange stages through host
memory; on the 8-GPU box the same code runs over NCCL).  Each rank runs BandPciam (forward of
its owned tiles; its interior pairs while the halo row's spectra arrive from rank-1 on a side
stream; then its boundary pairs), results are merged with gather_translations, and the merge
must be bit-identical to one whole-grid context (reading C16).  The in-library NCCL
transport cannot form a communicator with two ranks on one device; that it reports
STITCH_ERR_NCCL on every rank (instead of hanging) is checked too."""
import os
import socket

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

import torch.distributed as dist  # noqa: E402
import torch.multiprocessing as mp  # noqa: E402


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, n, m, H, W, transport, out):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import synthgrid
        from paper_conf_icpp_blattnerkcsbz14_b200.parallel import BandPciam, gather_translations
        torch.cuda.set_device(0)
        g = synthgrid.make_grid(n, m, H, W, seed=71)
        bp = BandPciam(n, m, H, W, rank, world, device=0, transport=transport)
        rows = g.tiles[bp.bd.row_begin: bp.bd.row_end]
        bp.load_rows(np.ascontiguousarray(rows))
        for _ in range(2):                     # second step replays the captured graphs
            bp.step_async()
            w, nn = bp.translations()
        w, nn = gather_translations(w, nn, bp.bd)
        if rank == 0:
            np.save(out + "_w.npy", w.view(np.uint8))
            np.save(out + "_n.npy", nn.view(np.uint8))
            out_flag = open(out + "_used_exchange", "w")
            out_flag.write(str(int(bp.use_exchange)))
            out_flag.close()
        bp.close()
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,transport", [(2, "torch"), (3, "torch"), (2, "recompute")])
def test_row_bands_over_torch_distributed_match_one_context(world, transport, tmp_path):
    import synthgrid
    from paper_conf_icpp_blattnerkcsbz14_b200 import PciamGrid
    n, m, H, W = 6, 5, 192, 256
    g = synthgrid.make_grid(n, m, H, W, seed=71)
    with PciamGrid(n, m, H, W) as pg:
        pg.load_grid(g.tiles)
        ref_w, ref_n = pg.compute_translations()
    out = str(tmp_path / "res")
    mp.spawn(_worker, args=(world, _free_port(), n, m, H, W, transport, out), nprocs=world,
             join=True)
    assert open(out + "_used_exchange").read() == str(int(transport != "recompute"))
    w = np.load(out + "_w.npy")
    nn = np.load(out + "_n.npy")
    assert w.tobytes() == ref_w.tobytes() and nn.tobytes() == ref_n.tobytes()


def _nccl_worker(rank, world, port, out):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_icpp_blattnerkcsbz14_b200 import StitchError
        from paper_conf_icpp_blattnerkcsbz14_b200.parallel import BandPciam
        torch.cuda.set_device(0)
        try:
            BandPciam(6, 5, 192, 256, rank, world, device=0, transport="library").close()
            status = 0
        except StitchError as e:
            status = e.status
        with open(f"{out}_{rank}", "w") as f:
            f.write(str(status))
    finally:
        dist.destroy_process_group()


@pytest.mark.timeout(300)
def test_library_nccl_transport_reports_error_on_shared_device(tmp_path):
    """stitch_init with an nccl_id: the library loads NCCL, joins the communicator -- which NCCL
    refuses for two ranks on one GPU -- and fails cleanly with STITCH_ERR_NCCL on both ranks."""
    out = str(tmp_path / "st")
    mp.spawn(_nccl_worker, args=(2, _free_port(), out), nprocs=2, join=True)
    assert [open(f"{out}_{k}").read() for k in range(2)] == ["5", "5"]
