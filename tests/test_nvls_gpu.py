"""the map exchange summed in the NVSwitch by toast_map_allreduce_nvls
(multimem.ld_reduce / multimem.st over torch symmetric memory's multicast mapping).

Only one GPU is reachable here, so this runs the world-size-1 case: the sum over one rank is the
buffer itself (bit-exact), through the real multicast mapping and the real kernel; it skips when
the device / driver has no multicast support.  The N > 1 arithmetic is the switch's add."""
import os
import socket

import pytest

torch = pytest.importorskip("torch")

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.fixture(scope="module")
def group():
    import torch.distributed as dist
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    torch.cuda.set_device(0)
    created = False
    if not dist.is_initialized():
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ["MASTER_PORT"] = str(_free_port())
        dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
        created = True
    yield dist.group.WORLD
    if created:
        dist.destroy_process_group()


def test_map_allreduce_nvls_world_one(group):
    from paper_conf_sc_demeurekktbb23_b200 import dist as tdist
    try:
        r = tdist.NvlsReducer(1 << 16, "cuda", group)
    except Exception as e:  # noqa: BLE001
        pytest.skip(f"no multicast / symmetric memory here: {type(e).__name__}: {e}")
    g = torch.Generator(device="cuda").manual_seed(7)
    for n in (1, 1000, 65536):  # ragged sizes, repeated calls
        x = torch.randn(n, dtype=torch.float64, device="cuda", generator=g)
        ref = x.clone()
        r.allreduce_(x)
        torch.cuda.synchronize()
        assert torch.equal(x, ref)
    # in place on the symmetric buffer, shaped like a packed map [n_submap][n_pix_submap][3]
    v = r.buf[: 4 * 1024 * 3].view(4, 1024, 3)
    v.copy_(torch.arange(v.numel(), dtype=torch.float64, device="cuda").view_as(v))
    r.allreduce_(v)
    torch.cuda.synchronize()
    assert torch.equal(v.flatten(), torch.arange(v.numel(), dtype=torch.float64, device="cuda"))
