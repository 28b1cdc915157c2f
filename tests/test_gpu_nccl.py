"""The NCCL transport of the z-slab halo exchange on one GPU.

NCCL refuses two ranks of one communicator on the same device, so this pool
(one GPU per box) cannot run the 2-rank exchange itself.  What it can run is
the exchange's own grouped call -- `nccl_group` in csrc/dist.cpp, the code that
issues ncclSend / ncclRecv for the halo planes -- on a 1-rank communicator
sending to itself: the dlopen'd entry points, their argument order, the FP64
datatype and the element counts are the ones the halo exchange uses, and the
received planes must equal the sent ones bit for bit.  The exchange's plane
offsets (halo_schedule) are pinned bitwise by the loopback transport
(test_gpu_parity.py, test_dist_hostlogic.py)."""
from __future__ import annotations

import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("no CUDA device", allow_module_level=True)

import paper_conf_ipps_rawatvsrps19_b200 as sdag  # noqa: E402


@pytest.fixture(scope="module")
def comm():
    uid = sdag.nccl_unique_id()
    c = sdag.nccl_comm_create(uid, 1, 0, torch.cuda.current_device())
    yield c
    sdag.nccl_comm_destroy(c)


@pytest.mark.parametrize("planes", [1, 2, 4])
def test_nccl_self_sendrecv_halo_planes_bitwise(comm, planes):
    ny, nx = 130, 258
    n = planes * ny * nx
    # integer-coded plane values (exact in FP64), plus signed zeros and a NaN payload
    src = torch.arange(n, dtype=torch.float64, device="cuda") * 0.5 - 7.0
    src[3] = -0.0
    src[5] = float("nan")
    dst = torch.full_like(src, 12345.0)
    s = torch.cuda.Stream()
    sdag.nccl_sendrecv(comm, 0, src, dst, stream=s)
    s.synchronize()
    assert torch.equal(src.view(torch.int64), dst.view(torch.int64))


def test_nccl_sendrecv_into_a_slab_ghost_region(comm):
    """the exchange's pattern: owned planes of one slab buffer into the ghost
    planes of another (pointer offsets inside one allocation)"""
    H, own, ny, nx = 2, 6, 40, 66
    a = torch.arange((own + 2 * H) * ny * nx, dtype=torch.float64, device="cuda").view(own + 2 * H, ny, nx)
    b = torch.full_like(a, -1.0)
    # lowest H owned planes of a -> ghost planes below b's owned planes
    sdag.nccl_sendrecv(comm, 0, a[H:2 * H], b[0:H])
    torch.cuda.synchronize()
    assert torch.equal(b[0:H], a[H:2 * H])
    assert torch.all(b[H:] == -1.0)


def test_nccl_sendrecv_rejects_bad_arguments(comm):
    x = torch.zeros(8, dtype=torch.float64, device="cuda")
    with pytest.raises(ValueError):
        sdag.nccl_sendrecv(comm, 0, x, torch.zeros(4, dtype=torch.float64, device="cuda"))
    with pytest.raises(sdag.SdagError):
        sdag.nccl_sendrecv(0, 0, x, x.clone())  # null communicator
