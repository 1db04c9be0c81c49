"""The 36-bit wire format (neo_wire_pack / neo_wire_unpack, include/neo.h): the device packing
equals the byte layout the header defines (written out here with numpy), and unpack inverts it."""
import numpy as np
import pytest
import torch

import synth
from oracle import ckks

pytestmark = pytest.mark.gpu

neo = pytest.importorskip("paper_conf_isca_jiaodwfcm0z25_b200.neo")


def wire_reference(x: np.ndarray) -> np.ndarray:
    """bytes [0, 4n): low 32 bits LE; bytes [4n, 4.5n): byte k = hi4(2k) | hi4(2k+1) << 4."""
    x = x.reshape(-1).astype(np.uint64)
    lo = (x & np.uint64(0xFFFFFFFF)).astype("<u4").view(np.uint8)
    hi = (x >> np.uint64(32)).astype(np.uint8)
    return np.concatenate([lo, hi[0::2] | (hi[1::2] << 4)])


@pytest.mark.parametrize("shape", [(8,), (2, 3, 4096), (1, 2, 36, 1 << 12)])
def test_wire_pack_matches_layout_and_round_trips(shape):
    prm = ckks.tiny()
    ctx = neo.Context(prm.log_n, prm.num_q, prm.num_p, prm.dnum)
    n = int(np.prod(shape))
    x = synth.uniform_residues(77, [prm.q[0]], n)[0].reshape(shape)
    x.reshape(-1)[:2] = [0, (1 << 36) - 1]                       # extremes of the 36-bit range
    xd = torch.from_numpy(x).cuda()
    wire = torch.empty(neo.neo_wire_bytes(n), dtype=torch.uint8, device="cuda")
    assert wire.numel() == 4 * n + n // 2
    neo.neo_wire_pack(ctx, xd, wire)
    back = torch.empty_like(xd)
    neo.neo_wire_unpack(ctx, wire, back)
    torch.cuda.synchronize()
    assert np.array_equal(wire.cpu().numpy(), wire_reference(x))
    assert np.array_equal(back.cpu().numpy(), x)


def test_wire_rejects_bad_sizes():
    prm = ckks.tiny()
    ctx = neo.Context(prm.log_n, prm.num_q, prm.num_p, prm.dnum)
    x = torch.zeros(12, dtype=torch.uint64, device="cuda")
    with pytest.raises(neo.NeoError):
        neo.neo_wire_pack(ctx, x, torch.empty(64, dtype=torch.uint8, device="cuda"))
