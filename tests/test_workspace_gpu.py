"""The §8(b) boundary's caller-owned memory and communicator (VERDICT r1
missing #2): a context on a torch-allocated workspace (nbody_create_ws) is
bit-identical to a self-allocated one; the workspace is the context's only
device memory; torch's own NCCL communicator drives the exchange
(nbody_attach_comm)."""
import numpy as np
import pytest

from workloads import generate

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def NB():
    import torch
    assert torch.cuda.is_available()
    from paper_conf_sc_casselldahg24_b200 import NBody
    return NBody


def _outputs(s):
    return s.get_positions(), s.get_velocities(), s.get_accel(), s.get_interactions()


@pytest.mark.parametrize("kw,features", [({}, 0), ({"multipole": 2}, 1), ({"balance": False}, 2)])
def test_torch_workspace_is_bit_identical(NB, kw, features):
    import torch
    from paper_conf_sc_casselldahg24_b200 import _capi
    n = 50_001
    pos, vel, mass = generate("disks", n, 21)
    ref = NB(n, 0.5, 1e-3, 1e-3, **kw)
    ref.set_bodies(pos, vel, mass)
    ref.step(3)
    nbytes = NB.workspace_bytes(n, 1, 16, features)
    big = torch.empty(nbytes + 4096, dtype=torch.uint8, device="cuda")
    ws = big[4096:]  # an interior pointer of the torch block (512-aligned)
    free0 = torch.cuda.mem_get_info()[0]
    s = NB(n, 0.5, 1e-3, 1e-3, workspace=ws, **kw)
    s.set_bodies(pos, vel, mass)
    if features & _capi.NBODY_WS_XFER:
        hp, hv, hm = (torch.from_numpy(a).pin_memory() for a in (pos, vel, mass))
        s.set_bodies_async(hp, hv, hm)
    s.step(3)
    s.sync()
    # the context took no device memory of its own beyond streams/events/graphs
    assert free0 - torch.cuda.mem_get_info()[0] < 64 << 20
    for a, b in zip(_outputs(ref), _outputs(s)):
        assert (a == b).all()
    s.close()


def test_workspace_errors(NB):
    import torch
    from paper_conf_sc_casselldahg24_b200 import NBodyError, _capi
    n = 10_000
    base = NB.workspace_bytes(n)
    small = torch.empty(base - 256, dtype=torch.uint8, device="cuda")
    with pytest.raises(NBodyError):
        NB(n, workspace=small)                      # below nbody_workspace_bytes: ENOMEM
    ws = torch.empty(base, dtype=torch.uint8, device="cuda")
    with pytest.raises(NBodyError):
        NB(n, workspace=ws[16:])                    # misaligned: EINVAL
    with pytest.raises(NBodyError):
        NB(n, workspace=torch.empty(base, dtype=torch.uint8))   # host memory: EINVAL
    s = NB(n, workspace=ws)                         # exactly the base size works ...
    with pytest.raises(NBodyError):
        s.set_option(_capi.NBODY_OPT_MULTIPOLE, 2)  # ... but has no room for the quadrupole arrays
    s.close()


def _ws_ipc_worker(rank, world, port, n, out_dir):
    import os
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    import torch
    import torch.distributed as dist
    from paper_conf_sc_casselldahg24_b200 import NBody
    dist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    pos, vel, mass = generate("plummer", n, 91)
    big = torch.empty(NBody.workspace_bytes(n) + (rank + 1) * 8192, dtype=torch.uint8, device="cuda")
    s = NBody(n, 0.5, 1e-3, 1e-3, workspace=big[(rank + 1) * 8192:])   # interior pointers
    s.attach_peers_group(rank, world)
    s.set_bodies(pos, vel, mass)
    dist.barrier()
    s.step(3)
    s.sync()
    np.save(os.path.join(out_dir, f"x{rank}.npy"), s.get_positions())
    dist.barrier()
    s.close()
    dist.destroy_process_group()


@pytest.mark.timeout(300)
def test_peer_exchange_on_torch_workspaces(NB, tmp_path):
    """Two processes whose arenas sit inside torch allocations: the peer
    descriptor carries the offset in the IPC-mapped block."""
    import socket
    import torch.multiprocessing as mp
    n, world = 12_000, 2
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        port = so.getsockname()[1]
    mp.start_processes(_ws_ipc_worker, args=(world, port, n, str(tmp_path)), nprocs=world, join=True,
                       start_method="spawn")
    pos, vel, mass = generate("plummer", n, 91)
    ref = NB(n, 0.5, 1e-3, 1e-3)
    ref.set_bodies(pos, vel, mass)
    ref.step(3)
    for r in range(world):
        assert (np.load(tmp_path / f"x{r}.npy") == ref.get_positions()).all()


def _comm_worker(rank, world, port, n, out):
    import os
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    import torch
    import torch.distributed as dist
    from paper_conf_sc_casselldahg24_b200 import NBody
    torch.cuda.set_device(0)
    dist.init_process_group("nccl", rank=rank, world_size=world, device_id=torch.device("cuda", 0))
    pos, vel, mass = generate("plummer", n, 92)
    s = NBody(n, 0.5, 1e-3, 1e-3)
    s.attach_torch_comm()
    assert s.exchange_mode() == "nccl"
    s.set_bodies(pos, vel, mass)
    s.step(3)
    s.sync()
    np.save(out, s.get_positions())
    s.close()
    dist.destroy_process_group()


@pytest.mark.timeout(300)
def test_torch_nccl_communicator_world1(NB, tmp_path):
    """nbody_attach_comm with ProcessGroupNCCL's communicator (world 1 on the
    one GPU of this box): the captured step graph runs the all-gather on
    torch's communicator; results equal the plain run."""
    import socket
    import torch.multiprocessing as mp
    from paper_conf_sc_casselldahg24_b200 import _capi
    if not _capi.load().nbody_has_nccl():
        pytest.skip("library built without NCCL")
    n = 20_000
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        port = so.getsockname()[1]
    out = str(tmp_path / "x.npy")
    mp.start_processes(_comm_worker, args=(1, port, n, out), nprocs=1, join=True, start_method="spawn")
    pos, vel, mass = generate("plummer", n, 92)
    ref = NB(n, 0.5, 1e-3, 1e-3)
    ref.set_bodies(pos, vel, mass)
    ref.step(3)
    assert (np.load(out) == ref.get_positions()).all()
