"""Tile blocks that stack several images (Plan::NI > 1: the staged input box and the
output store box carry NI images, lanes map to (image, row, tile)). The planner picks
NI > 1 for small images at full size (28x28 configs, tests/test_gpu_fullsize.py); here
I2CW_NI forces it on the small parity cases, including a ragged last image group
(N not a multiple of NI: the TMA zero-fills the missing images and clips their stores).
The variable is read once per process, so the cases run in a subprocess."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.parametrize("ni", ["2", "3"])
def test_multi_image_parity_subset(ni):
    env = dict(os.environ, I2CW_NI=ni)
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-p", "no:cacheprovider",
                        os.path.join(ROOT, "tests", "test_gpu_parity.py"),
                        "-k", "r_sweep_same_pad or small_k or pads or rect or deconv_pad"],
                       cwd=ROOT, env=env, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-2000:]
