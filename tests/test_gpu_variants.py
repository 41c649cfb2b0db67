"""Runtime-selectable kernel variants (environment knobs read once per process, so each
runs the parity subset in a subprocess of its own):
  MOE_SWAP_NP1/2=2  prefill grouped GEMMs on clusters of 2 CTA pairs with multicast token boxes
                    (opt-in: measured slower on a B200, profiles/r02/swap_np.txt)
  MOE_FD_CSIZE=C    the fused decode stream split over clusters of C CTAs, each cluster
                    taking several units from the queue (the cost model picks C otherwise)"""
import os
import subprocess
import sys

import pytest
import torch

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.parametrize("env,select", [
    ({"MOE_SWAP_NP1": "2", "MOE_SWAP_NP2": "2"}, "small_layer or swap_pair or prefill_8k"),
    ({"MOE_FD_CSIZE": "2"}, "decode_shapes or fused_decode"),
    ({"MOE_FD_CSIZE": "4"}, "decode_shapes or fused_decode or mid_size_decode"),
    ({"MOE_FD_CSIZE": "8"}, "decode_shapes or fused_decode"),
])
def test_variant_parity(env, select):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    e = dict(os.environ, **env)
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-p", "no:cacheprovider",
                        os.path.join(ROOT, "tests", "test_gpu_parity.py"), "-k", select],
                       cwd=ROOT, env=e, capture_output=True, text=True, timeout=900)
    tail = "\n".join((r.stdout + r.stderr).strip().splitlines()[-15:])
    assert r.returncode == 0, f"{env}: {tail}"
