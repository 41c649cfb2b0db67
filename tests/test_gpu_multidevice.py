"""Two layers on two devices in one process (skips with fewer than 2 GPUs).

The >48 KB shared-memory kernels need their cudaFuncSetAttribute opt-in per device context
(kernels.h set_kernel_attr); this runs every kernel family on device 0 and device 1 and checks
the two devices agree.  Prefill (grouped GEMMs) is deterministic, so it must match bitwise; the
decode stream sums in fp32 atomics (R22), so it matches to fp32 rounding.
"""
import pytest
import torch

from inputs.presets import SMALL
from inputs.synthetic import make_tokens, make_weights

pytestmark = pytest.mark.gpu


def _need_two():
    if not torch.cuda.is_available() or torch.cuda.device_count() < 2:
        pytest.skip("needs 2 CUDA devices")


@pytest.mark.parametrize("name", ["v3_s", "v3_s_fp4"])
def test_two_devices_agree(name):
    _need_two()
    from paper_conf_sosp_chenxztwdcylqzo25_b200 import moe
    p = SMALL[name]
    w = make_weights(p, "cpu")
    outs = []
    for dev in (0, 1):
        wd = w.to(f"cuda:{dev}")
        layer = moe.MoELayer(p, wd, max_tokens=300, device=dev)
        x, r = make_tokens(p, 300, f"cuda:{dev}")
        y_pf = layer.forward(x, r)
        y_dc = layer.forward(x[:3].contiguous(), r[:3].contiguous())
        torch.cuda.synchronize(dev)
        outs.append((y_pf.cpu(), y_dc.cpu()))
        layer.close()
    assert torch.equal(outs[0][0], outs[1][0])
    torch.testing.assert_close(outs[0][1].float(), outs[1][1].float(), rtol=2e-2, atol=2e-2)
