"""the map exchange summed in the NVSwitch by toast_map_allreduce_nvls
(multimem.ld_reduce / multimem.st over torch symmetric memory's multicast mapping).

Only one GPU is reachable here, so this runs the world-size-1 case: the sum over one rank is the
buffer itself (bit-exact), through the real multicast mapping and the real kernel; it skips when
the device / driver has no multicast support.  The N > 1 arithmetic is the switch's add."""
import ctypes
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


def _ck(r):
    from cuda.bindings import driver as cu
    err = r[0] if isinstance(r, tuple) else r
    if err != cu.CUresult.CUDA_SUCCESS:
        raise RuntimeError(f"CUDA driver: {err}")
    if isinstance(r, tuple):
        return r[1] if len(r) == 2 else r[1:]
    return None


class _DevArray:
    def __init__(self, ptr, n):
        self.__cuda_array_interface__ = {"shape": (n,), "typestr": "<f8", "data": (int(ptr), False), "version": 3}


def test_map_allreduce_nvls_on_a_driver_multicast_object():
    """The kernel on a multicast object the test builds itself with the driver API (one device,
    no shareable handle): every element of ragged slices comes back as the 1-rank sum (itself)."""
    cu = pytest.importorskip("cuda.bindings.driver")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    torch.cuda.set_device(0)
    torch.cuda.synchronize()
    _ck(cu.cuInit(0))
    dev = _ck(cu.cuDeviceGet(0))
    if not _ck(cu.cuDeviceGetAttribute(cu.CUdevice_attribute.CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, dev)):
        pytest.skip("device reports no multicast support")
    n = 300_001
    mcp = cu.CUmulticastObjectProp()
    mcp.numDevices = 1
    mcp.handleTypes = cu.CUmemAllocationHandleType.CU_MEM_HANDLE_TYPE_NONE
    mcp.size = n * 8
    gran = _ck(cu.cuMulticastGetGranularity(mcp, cu.CUmulticastGranularity_flags.CU_MULTICAST_GRANULARITY_RECOMMENDED))
    size = (n * 8 + gran - 1) // gran * gran
    mcp.size = size
    try:
        mc = _ck(cu.cuMulticastCreate(mcp))
        _ck(cu.cuMulticastAddDevice(mc, dev))
    except RuntimeError as e:
        pytest.skip(f"cuMulticastCreate on one device: {e}")
    prop = cu.CUmemAllocationProp()
    prop.type = cu.CUmemAllocationType.CU_MEM_ALLOCATION_TYPE_PINNED
    prop.location.type = cu.CUmemLocationType.CU_MEM_LOCATION_TYPE_DEVICE
    prop.location.id = 0
    mem = _ck(cu.cuMemCreate(size, prop, 0))
    _ck(cu.cuMulticastBindMem(mc, 0, mem, 0, size, 0))
    acc = cu.CUmemAccessDesc()
    acc.location.type = cu.CUmemLocationType.CU_MEM_LOCATION_TYPE_DEVICE
    acc.location.id = 0
    acc.flags = cu.CUmemAccess_flags.CU_MEM_ACCESS_FLAGS_PROT_READWRITE
    uc_va = _ck(cu.cuMemAddressReserve(size, gran, 0, 0))
    _ck(cu.cuMemMap(uc_va, size, 0, mem, 0))
    _ck(cu.cuMemSetAccess(uc_va, size, [acc], 1))
    mc_va = _ck(cu.cuMemAddressReserve(size, gran, 0, 0))
    _ck(cu.cuMemMap(mc_va, size, 0, mc, 0))
    _ck(cu.cuMemSetAccess(mc_va, size, [acc], 1))
    try:
        from paper_conf_sc_demeurekktbb23_b200 import binding
        lib = binding.load()
        x = torch.as_tensor(_DevArray(int(uc_va), n), device="cuda")
        g = torch.Generator(device="cuda").manual_seed(11)
        ref = torch.randn(n, dtype=torch.float64, device="cuda", generator=g)
        st = torch.cuda.current_stream()
        for m in (1, 4097, n):
            x.copy_(ref)
            rc = lib.toast_map_allreduce_nvls(ctypes.c_void_p(int(mc_va)), m, None, 0, 1,
                                              ctypes.c_void_p(st.cuda_stream))
            assert rc == 0, lib.toast_last_error()
            torch.cuda.synchronize()
            assert torch.equal(x, ref)
    finally:
        torch.cuda.synchronize()
        for va in (uc_va, mc_va):
            cu.cuMemUnmap(va, size)
            cu.cuMemAddressFree(va, size)
        cu.cuMulticastUnbind(mc, dev, 0, size)
        cu.cuMemRelease(mem)
        cu.cuMemRelease(mc)
